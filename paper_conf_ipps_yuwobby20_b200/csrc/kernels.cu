// kernels.cu — sm_100a kernels of the IDFG fixed point.
//
// One warp processes one worklist node (Alg. 3 l.9-15): it reads the
// node's fact block IN(src) (MAT) with coalesced 8-byte-per-lane loads,
// applies the node's transfer function on the fly (GEN_KILL, Alg. 3 l.10), maps the result
// through each out-edge (SEARCH, l.11; edge transforms of DESIGN.md §3 C3) and ORs it into
// IN(dst) with 64-bit atomicOr, skipping words whose bits are already present (a plain,
// possibly stale load first: IN only grows, so a stale read never hides a needed OR).
// update() (l.14) = "some word gained a bit" (warp vote).  Destinations that grew, or were
// never queued (first-reach rule, DESIGN.md §3 A5), are appended to the next round's
// class-segmented worklist (GRP, l.7) behind a per-node round stamp (atomicMax test-and-set),
// which de-duplicates exactly like MER's merge (Fig. 7).
//
// The round loop runs inside one persistent cooperative kernel with a grid barrier per
// round (no host round trip), or as one launch per round (loop_mode 1).
#include <cooperative_groups.h>

#include "internal.cuh"

namespace gd {
namespace {

constexpr unsigned FULL = 0xffffffffu;

struct Acc {              // per-lane counters, reduced once per kernel
  unsigned long long nz;  // non-zero edge words written (x16 bytes in the touched model)
  unsigned long long nzx; // non-zero IN(src) words read (x8)
  unsigned long long h;   // heap words gathered by DOUBLE kinds (x8)
  unsigned long long atom;
  unsigned long long dense;   // dense-model bytes (lane 0 only)
  unsigned long long fixed;   // per-visit constant bytes (lane 0 only)
};

struct WarpScratch {
  uint64_t gen[MAXW];     // generated row (replace / or-in)
  uint64_t rv[MAXW];      // FSTORE base row v
  uint64_t rw[MAXW];      // FSTORE / FLOAD value row w
};

__device__ __forceinline__ uint64_t warp_or64(uint64_t v) {
  uint32_t lo = __reduce_or_sync(FULL, (uint32_t)v);
  uint32_t hi = __reduce_or_sync(FULL, (uint32_t)(v >> 32));
  return ((uint64_t)hi << 32) | lo;
}

__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {   // splitmix64 finaliser (C8)
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

// global-part-relative row of heap slot (instance in column c, field f) or -1 (C1)
__device__ __forceinline__ int heap_row_rel(const Dev& D, const ModRec& md, uint32_t c, uint32_t f) {
  int t = D.col_type[md.col_off + c];
  if (t < 0) return -1;
  uint32_t a = D.tf_ptr[t], b = D.tf_ptr[t + 1];
  for (uint32_t k = a; k < b; ++k)
    if (D.tf[k] == f) return (int)(D.col_hbase[md.col_off + c] + (k - a));
  return -1;
}

// IN(dst)[w] |= y; returns whether IN(dst) gained a bit (update(), A6)
__device__ __forceinline__ bool or_into(uint64_t* p, uint64_t y, Acc& acc) {
  if (!y) return false;
  acc.nz++;
  uint64_t cur = *p;                  // may be stale (subset of the truth): safe
  if (!(y & ~cur)) return false;
  uint64_t old = atomicOr((unsigned long long*)p, (unsigned long long)y);
  acc.atom++;
  return (y & ~old) != 0;
}

// Y[w] = f_src(X)[w] (DESIGN.md §3 C2), X[w] returned in x
__device__ __forceinline__ uint64_t y_word(const Dev& D, const uint64_t* __restrict__ X, uint32_t w,
                                           uint32_t logW, int mode, int t, uint32_t L,
                                           const ModRec& md, uint32_t f, const WarpScratch& ws,
                                           uint64_t& x) {
  x = X[w];
  if (mode == 0) return x;
  const uint32_t r = w >> logW, j = w & ((1u << logW) - 1);
  if (mode == 1) return (int)r == t ? ws.gen[j] : x;            // X \ K(v) ∪ gen
  if (mode == 2) return (int)r == t ? (x | ws.gen[j]) : x;      // weak static store
  if (r >= L + md.n_stat) {                                      // FSTORE: heap rows (o1, f)
    const uint32_t g = r - L;
    if (D.grow_field[md.grow_off + g] == (int)f) {
      const int c = D.grow_col[md.grow_off + g];                 // o1 (never NULL)
      if ((ws.rv[c >> 6] >> (c & 63)) & 1ull) return x | ws.rw[j];
    }
  }
  return x;
}

// Append the candidate destinations held by the warp's lanes to the next worklist.
__device__ __forceinline__ void flush_pushes(const Dev& D, int lane, bool active, uint32_t dst,
                                             bool grew, uint32_t round, uint32_t nxt) {
  bool push = false;
  int cls = -1;
  if (active) {
    bool want = grew || (D.stamp[dst] == 0);               // grew, or first reach (A5)
    if (want) {
      uint32_t old = atomicMax(&D.stamp[dst], round + 1);  // test-and-set: de-duplicates (MER)
      push = old < round + 1;
    }
    if (push) cls = D.nodes[dst].cls;
  }
  unsigned pm = __ballot_sync(FULL, push);
  while (pm) {                                             // warp-aggregated append per class
    const int leader = __ffs(pm) - 1;
    const int c = __shfl_sync(FULL, cls, leader);
    const unsigned same = __ballot_sync(FULL, push && cls == c);
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(&D.counts[nxt * CNT_STRIDE + c], (uint32_t)__popc(same));
    base = __shfl_sync(FULL, base, leader);
    if (push && cls == c) {
      const uint32_t rank = __popc(same & ((1u << lane) - 1));
      D.queue[(size_t)nxt * D.n_nodes + D.seg[c] + base + rank] = dst;
    }
    pm &= ~same;
  }
}

// One worklist node, one warp (Alg. 3 l.9-15).
__device__ void process_node(const Dev& D, uint32_t n, uint32_t round, uint32_t nxt, int lane,
                             WarpScratch& ws, Acc& acc) {
  const uint32_t e0 = D.row_ptr[n], e1 = D.row_ptr[n + 1];
  if (lane == 0) acc.fixed += sizeof(NodeRec) + 8 + 8ull * (e1 - e0) + 8;
  if (e0 == e1) return;                                    // no successor: nothing to propagate
  const NodeRec R = D.nodes[n];
  const MethRec mr = D.meths[R.method];
  const ModRec md = D.mods[mr.module];
  const uint32_t logW = md.logW, W = md.W, L = mr.n_locals;
  const uint32_t B = (L + md.n_glob) << logW;
  const uint64_t* __restrict__ X = D.facts + R.off;

  // ---- GEN_KILL setup (a4): mode 0 identity, 1 replace row t, 2 or into row t, 3 FSTORE
  int mode = 0, t = -1;
  uint32_t f = 0;
  switch (R.kind) {
    case GK_PRIM:
      mode = 1; t = R.r0;
      if (lane < (int)W) ws.gen[lane] = 0;
      break;
    case GK_CONST: case GK_NEW:
      mode = 1; t = R.r0;
      if (lane < (int)W) ws.gen[lane] = ((R.r3 >> 6) == lane) ? (1ull << (R.r3 & 63)) : 0ull;
      break;
    case GK_COPY: case GK_SLOAD: case GK_RETV:
      mode = 1; t = R.r0;
      if (lane < (int)W) ws.gen[lane] = X[((uint64_t)R.r1 << logW) + lane];
      break;
    case GK_SSTORE:
      mode = 2; t = R.r0;
      if (lane < (int)W) ws.gen[lane] = X[((uint64_t)R.r1 << logW) + lane];
      break;
    case GK_FLOAD: case GK_ALOAD: {          // v = w.f: OR of heap rows (o1, f), o1 ∈ row w
      mode = 1; t = R.r0; f = (uint32_t)R.r2;
      if (lane < (int)W) ws.rw[lane] = X[((uint64_t)R.r1 << logW) + lane];
      __syncwarp();
      uint64_t a[MAXW];
#pragma unroll
      for (int j = 0; j < MAXW; ++j) a[j] = 0;
      for (uint32_t c = lane; c < md.n_cols; c += 32) {
        if (c == 0 || !((ws.rw[c >> 6] >> (c & 63)) & 1ull)) continue;   // NULL has no fields
        const int hr = heap_row_rel(D, md, c, f);
        if (hr < 0) continue;
        const uint64_t* H = X + ((uint64_t)(L + hr) << logW);
#pragma unroll
        for (int j = 0; j < MAXW; ++j)
          if (j < (int)W) a[j] |= H[j];
        acc.h += W;
      }
#pragma unroll
      for (int j = 0; j < MAXW; ++j) {
        if (j < (int)W) {
          const uint64_t v = warp_or64(a[j]);
          if (lane == 0) ws.gen[j] = v;
        }
      }
      break;
    }
    case GK_FSTORE: case GK_ASTORE:          // v.f = w (weak)
      mode = 3; f = (uint32_t)R.r2;
      if (lane < (int)W) {
        ws.rv[lane] = X[((uint64_t)R.r0 << logW) + lane];
        ws.rw[lane] = X[((uint64_t)R.r1 << logW) + lane];
      }
      break;
    default:
      break;                                 // NOP/ENTRY/EXIT/RETSITE/CALL: identity
  }
  __syncwarp();

  // ---- SEARCH + union/update over the out-edges (a5)
  uint32_t cand_dst = 0;
  bool cand_grew = false;
  unsigned long long dense = 8ull * B + 8ull * acc.h;
  for (uint32_t e = e0; e < e1; ++e) {
    const Edge E = D.edges[e];
    const uint32_t kind = E.info & 3u, xid = E.info >> 2;
    const uint32_t dst = E.dst;
    const NodeRec RD = D.nodes[dst];
    uint64_t* Z = D.facts + RD.off;
    const bool first = (e == e0);
    bool grew = false;
    if (kind == GE_INTRA || kind == GE_C2R) {
      const int kill = (kind == GE_C2R) ? R.r0 : -1;       // C2R drops lhs(c)
      for (uint32_t w = lane; w < B; w += 32) {
        uint64_t x;
        uint64_t y = y_word(D, X, w, logW, mode, t, L, md, f, ws, x);
        if (first) acc.nzx += (x != 0);
        if (kill >= 0 && (int)(w >> logW) == kill) y = 0;
        grew |= or_into(Z + w, y, acc);
      }
      dense += 16ull * B;
    } else if (xid == 0) {                                 // CALL / RET inside one module
      const MethRec mt = D.meths[RD.method];
      const uint32_t Lt = mt.n_locals, Bt = (Lt + md.n_glob) << logW;
      const uint32_t a0 = (kind == GE_CALL) ? D.arg_ptr[n] : 0;
      for (uint32_t w = lane; w < Bt; w += 32) {
        const uint32_t r = w >> logW, j = w & (W - 1);
        int src;
        if (r < Lt) {
          if (kind == GE_CALL) src = (r < mt.n_params) ? D.args[a0 + r] : -1;   // param_j <- arg_j
          else src = ((int)r == RD.r0) ? (int)(L - 1) : -1;                   // lhs(c) <- RET
        } else {
          src = (int)(L + (r - Lt));                                           // globals
        }
        if (src < 0) continue;
        const uint64_t y = X[((uint64_t)src << logW) + j];   // CALL/EXIT transfers are identity
        if (first) acc.nzx += (y != 0);
        grew |= or_into(Z + w, y, acc);
      }
      dense += 16ull * Bt;
    } else {                                               // CALL / RET across modules: π
      const XRec xr = D.xrecs[xid];
      const MethRec mt = D.meths[RD.method];
      const ModRec mdt = D.mods[mt.module];
      const uint32_t Lt = mt.n_locals, rows_t = Lt + mdt.n_glob, logWt = mdt.logW;
      const uint32_t a0 = (kind == GE_CALL) ? D.arg_ptr[n] : 0;
      for (uint32_t r = lane; r < rows_t; r += 32) {
        int src;
        if (r < Lt) {
          if (kind == GE_CALL) src = (r < mt.n_params) ? D.args[a0 + r] : -1;
          else src = ((int)r == RD.r0) ? (int)(L - 1) : -1;
        } else {
          const int gs = D.rowmap[xr.rowmap_off + (r - Lt)];
          src = gs < 0 ? -1 : (int)(L + gs);
        }
        if (src < 0) continue;
        uint64_t out[MAXW];
#pragma unroll
        for (int q = 0; q < MAXW; ++q) out[q] = 0;
        for (uint32_t j = 0; j < W; ++j) {
          uint64_t v = X[((uint64_t)src << logW) + j];
          if (first) acc.nzx += (v != 0);
          while (v) {
            const int b = __ffsll((long long)v) - 1;
            v &= v - 1;
            const int cd = D.colmap[xr.colmap_off + j * 64 + b];
            if (cd < 0) continue;
#pragma unroll
            for (int q = 0; q < MAXW; ++q)
              if (q == (cd >> 6)) out[q] |= 1ull << (cd & 63);
          }
        }
#pragma unroll
        for (int q = 0; q < MAXW; ++q)
          if (q < (int)mdt.W) grew |= or_into(Z + ((uint64_t)r << logWt) + q, out[q], acc);
      }
      dense += 16ull * ((uint64_t)rows_t << logWt);
    }
    grew = __any_sync(FULL, grew);
    const int slot = (int)((e - e0) & 31u);
    if (lane == slot) { cand_dst = dst; cand_grew = grew; }
    if (slot == 31 || e + 1 == e1) {
      flush_pushes(D, lane, lane <= slot, cand_dst, cand_grew, round, nxt);
    }
  }
  if (lane == 0) acc.dense += dense;
}

__device__ __forceinline__ void grid_sync(uint32_t* bar, uint32_t nblocks) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile uint32_t* vgen = bar + 1;
    const uint32_t gen = *vgen;
    __threadfence();
    const uint32_t arrived = atomicAdd(bar, 1u);
    if (arrived == nblocks - 1) {
      atomicExch(bar, 0u);
      __threadfence();
      atomicAdd(bar + 1, 1u);
    } else {
      while (*vgen == gen) __nanosleep(20);
    }
    __threadfence();                       // acquire: later loads see other SMs' writes
  }
  __syncthreads();
}

__device__ __forceinline__ void flush_acc(const Dev& D, Acc& acc) {
  unsigned long long ab = 16ull * acc.nz + 8ull * acc.nzx + 8ull * acc.h + acc.fixed;
  ab = warp_sum64(ab);
  const unsigned long long at = warp_sum64(acc.atom);
  const unsigned long long de = warp_sum64(acc.dense + acc.fixed);
  if ((threadIdx.x & 31) == 0 && (ab | at | de)) {
    atomicAdd(&D.stats->alg_bytes, ab);
    atomicAdd(&D.stats->atomics, at);
    atomicAdd(&D.stats->dense_bytes, de);
  }
}

// Process every item of round `round` with warps gw, gw+nw, ...; returns total items.
__device__ __forceinline__ uint32_t run_round(const Dev& D, uint32_t round, uint32_t gw, uint32_t nw,
                                              int lane, WarpScratch& ws, Acc& acc) {
  const uint32_t cur = round % 3, nxt = (round + 1) % 3, clr = (round + 2) % 3;
  if (D.bar[2]) return 0;                 // an earlier round found the worklist empty
  uint32_t pre[NCLS + 1];
  pre[0] = 0;
#pragma unroll
  for (int c = 0; c < NCLS; ++c) pre[c + 1] = pre[c] + D.counts[cur * CNT_STRIDE + c];
  const uint32_t total = pre[NCLS];
  if (total == 0) {                       // fixed point reached (Alg. 1 l.10)
    if (blockIdx.x == 0 && threadIdx.x == 0) D.bar[2] = 1;
    return 0;
  }
  if (D.max_rounds && round > D.max_rounds) return total;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
#pragma unroll
    for (int c = 0; c < NCLS; ++c) D.counts[clr * CNT_STRIDE + c] = 0;
    D.stats->rounds += 1;
    D.stats->visits += total;
    D.stats->hist[total <= 32 ? 0 : (total <= 64 ? 1 : 2)] += 1;
  }
  for (uint32_t item = gw; item < total; item += nw) {
    int c = 0;
    while (item >= pre[c + 1]) ++c;
    const uint32_t n = D.queue[(size_t)cur * D.n_nodes + D.seg[c] + (item - pre[c])];
    process_node(D, n, round, nxt, lane, ws, acc);
  }
  return total;
}

__global__ void __launch_bounds__(THREADS, 2) k_fixpoint(Dev D) {
  __shared__ WarpScratch ws_all[WARPS];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * WARPS + wib, nw = gridDim.x * WARPS;
  Acc acc = {};
  for (uint32_t round = 1;; ++round) {
    const uint32_t total = run_round(D, round, gw, nw, lane, ws_all[wib], acc);
    if (total == 0) break;
    if (D.max_rounds && round > D.max_rounds) {
      if (blockIdx.x == 0 && threadIdx.x == 0) D.stats->limit_hit = 1;
      break;
    }
    grid_sync(D.bar, gridDim.x);
  }
  flush_acc(D, acc);
}

__global__ void __launch_bounds__(THREADS, 2) k_round(Dev D, uint32_t round) {
  __shared__ WarpScratch ws_all[WARPS];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * WARPS + wib, nw = gridDim.x * WARPS;
  Acc acc = {};
  const uint32_t total = run_round(D, round, gw, nw, lane, ws_all[wib], acc);
  if (total && D.max_rounds && round > D.max_rounds && blockIdx.x == 0 && threadIdx.x == 0)
    D.stats->limit_hit = 1;
  flush_acc(D, acc);
}

// (a2) seed round 1 with the component entries (Alg. 1 l.9)
__global__ void k_seed(Dev D) {
  const int lane = threadIdx.x & 31;
  for (uint32_t i0 = 0; i0 < D.n_entries; i0 += 32) {
    const uint32_t i = i0 + lane;
    const bool act = i < D.n_entries;
    flush_pushes(D, lane, act, act ? D.entries[i] : 0, true, 0u, 1u);
  }
}

// (a7) per-node digests d(n) = Σ mix64(mix64(n) ^ (slot<<32 | inst)) (C8)
__global__ void __launch_bounds__(256) k_digest(Dev D) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < D.n_nodes; n += nw) {
    const NodeRec R = D.nodes[n];
    const MethRec mr = D.meths[R.method];
    const ModRec md = D.mods[mr.module];
    const uint32_t logW = md.logW, L = mr.n_locals, B = (L + md.n_glob) << logW;
    const uint64_t* X = D.facts + R.off;
    const uint64_t hn = mix64((uint64_t)(n - D.app_node_base[R.app]));
    unsigned long long s = 0;
    for (uint32_t w = lane; w < B; w += 32) {
      uint64_t x = X[w];
      if (!x) continue;
      const uint32_t r = w >> logW, j = w & ((1u << logW) - 1);
      const uint64_t slot = r < L ? (uint64_t)(mr.local_base + r) : (uint64_t)D.grow_gid[md.grow_off + r - L];
      while (x) {
        const int b = __ffsll((long long)x) - 1;
        x &= x - 1;
        const uint64_t o = D.col_gid[md.col_off + j * 64 + b];
        s += mix64(hn ^ ((slot << 32) | o));
      }
    }
    s = warp_sum64(s);
    if (lane == 0) {
      D.node_digest[n] = s;
      atomicAdd(&D.app_digest[R.app], s);
    }
  }
}

__global__ void k_popc(Dev D, uint32_t n0, uint32_t n1, uint64_t* out) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = n0 + blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < n1; n += nw) {
    const NodeRec R = D.nodes[n];
    const MethRec mr = D.meths[R.method];
    const ModRec md = D.mods[mr.module];
    const uint32_t B = (mr.n_locals + md.n_glob) << md.logW;
    unsigned long long c = 0;
    for (uint32_t w = lane; w < B; w += 32) c += __popcll(D.facts[R.off + w]);
    c = warp_sum64(c);
    if (lane == 0) out[n - n0] = c;
  }
}

// bits of IN(n) -> ascending (slot gid << 32 | inst gid): row-major order is ascending because
// rows are locals < statics < heap in gid order and columns are sorted instance gids.
__global__ void k_expand(Dev D, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = n0 + blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < n1; n += nw) {
    const NodeRec R = D.nodes[n];
    const MethRec mr = D.meths[R.method];
    const ModRec md = D.mods[mr.module];
    const uint32_t logW = md.logW, L = mr.n_locals, B = (L + md.n_glob) << logW;
    uint64_t base = ptr[n - n0];
    for (uint32_t w0 = 0; w0 < B; w0 += 32) {
      const uint32_t w = w0 + lane;
      uint64_t x = w < B ? D.facts[R.off + w] : 0;
      const uint32_t c = __popcll(x);
      uint32_t incl = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += v;
      }
      uint64_t pos = base + incl - c;
      if (x) {
        const uint32_t r = w >> logW, j = w & ((1u << logW) - 1);
        const uint64_t slot = r < L ? (uint64_t)(mr.local_base + r) : (uint64_t)D.grow_gid[md.grow_off + r - L];
        while (x) {
          const int b = __ffsll((long long)x) - 1;
          x &= x - 1;
          pairs[pos++] = (slot << 32) | D.col_gid[md.col_off + j * 64 + b];
        }
      }
      base += __shfl_sync(FULL, incl, 31);
    }
  }
}

}  // namespace

cudaError_t launch_seed(const Dev& D, cudaStream_t s) {
  k_seed<<<1, 32, 0, s>>>(D);
  return cudaGetLastError();
}

int fixpoint_max_blocks(int device) {
  int sms = 0, occ = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_fixpoint, THREADS, 0);
  return sms * (occ > 0 ? occ : 1);
}

cudaError_t launch_fixpoint(const Dev& D, uint32_t blocks, cudaStream_t s) {
  Dev d = D;
  void* args[] = {&d};
  return cudaLaunchCooperativeKernel((const void*)k_fixpoint, dim3(blocks), dim3(THREADS), args, 0, s);
}

cudaError_t launch_round(const Dev& D, uint32_t round, uint32_t blocks, cudaStream_t s) {
  k_round<<<blocks, THREADS, 0, s>>>(D, round);
  return cudaGetLastError();
}

cudaError_t launch_digest(const Dev& D, cudaStream_t s) {
  uint32_t blocks = (D.n_nodes + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks == 0) blocks = 1;
  k_digest<<<blocks, 256, 0, s>>>(D);
  return cudaGetLastError();
}

cudaError_t launch_popc(const Dev& D, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s) {
  uint32_t blocks = (n1 - n0 + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks == 0) blocks = 1;
  k_popc<<<blocks, 256, 0, s>>>(D, n0, n1, out);
  return cudaGetLastError();
}

cudaError_t launch_expand(const Dev& D, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs,
                          cudaStream_t s) {
  uint32_t blocks = (n1 - n0 + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks == 0) blocks = 1;
  k_expand<<<blocks, 256, 0, s>>>(D, n0, n1, ptr, pairs);
  return cudaGetLastError();
}

}  // namespace gd
