// kernels.cu — sm_100a kernels of the IDFG fixed point.
//
// One warp processes one work item = (node, chunk of its out-edges) (Alg. 3 l.9-15,
// PAPER.md:751-766): it reads the node's fact block IN(src) (MAT) with
// coalesced 8-byte-per-lane loads issued together with the edge records, applies the node's
// transfer function on the fly (GEN_KILL, Alg. 3 l.10), maps the result through each out-edge
// (SEARCH, l.11; edge transforms of DESIGN.md §3 C3) and ORs it into IN(dst) with
// fire-and-forget 64-bit RED.OR, only for words whose bits are missing (a plain, possibly
// stale load first: IN only grows, so a stale read never hides a needed OR, it can only
// over-report growth, which costs a duplicate push).  update() (l.14) = "some word had a
// missing bit" (warp vote).  Destinations that grew, or were never queued (first-reach rule,
// DESIGN.md §3 A5), are appended to the next round's class-segmented worklist (GRP, l.7)
// behind a per-node round stamp (atomicMax test-and-set) that de-duplicates like MER's merge
// (Fig. 7).  Appends are staged per CTA in shared memory and published
// with one global atomic per class per CTA at the end of the round.
//
// The round loop runs inside one persistent cooperative kernel with a grid barrier per
// round (no host round trip), or as one launch per round (loop_mode 1).
#include "internal.cuh"

namespace gd {
namespace {

#ifndef GD_MINB
#define GD_MINB 3              // resident CTAs per SM the fixed-point kernels are compiled for
#endif
#ifndef GD_MINB_WIDE
#define GD_MINB_WIDE GD_MINB   // ... for wide batches (4: measured flat, profiles/r02_ab_knobs.log)
#endif
#ifndef GD_MINB_HI
#define GD_MINB_HI 4           // ... for large narrow batches (Dev::hiocc)
#endif

constexpr unsigned FULL = 0xffffffffu;
constexpr int KW = 4;          // words per lane per chunk of a fact block (loads issued together)
constexpr int SCAP = 448 * THREADS / 256;   // staged queue entries per class per CTA (overflow goes global)
#ifndef GD_CONT_DEPTH
#define GD_CONT_DEPTH 8        // longest depth-first continuation per queued item (0 = off)
#endif
#ifndef GD_CONT_DEPTH_NARROW
#define GD_CONT_DEPTH_NARROW 3 // ... in narrow batches (sweeps: small 1.51 / 1.30 / 1.24 / 1.26 ms at 8 / 4 / 3 / 2, corpus flat)
#endif
#ifndef GD_CONT_LOAD
#define GD_CONT_LOAD 4         // continuation allowed in rounds with < GD_CONT_LOAD/4 items per warp
#endif
#ifndef GD_INL
#define GD_INL 1               // chunk-0 INTRA/C2R edges read from the inline record (one hop less)
#endif
#ifndef GD_PRE
#define GD_PRE 1               // inline path: load IN(dst) of the first two edges with IN(src)
#endif
#ifndef GD_PRE2
#define GD_PRE2 1              // ... and of the second edge
#endif
#ifndef GD_BAR_NS
#define GD_BAR_NS 20           // grid barrier: __nanosleep between polls of the generation word
#endif
#ifndef GD_CD_HI
#define GD_CD_HI 0             // narrow continuation compiled into the 4-CTA/SM (heavy-round) build too
#endif
#ifndef GD_PF
#define GD_PF 0                // two-stage prefetch pipeline across the items of a warp (run_round):
                               // +9 % on corpus200 (profiles/r02_ab_prefetch.log), off
#endif
#ifndef GD_PAIR
#define GD_PAIR 0              // heavy rounds: two inline items per warp (half-warp each); measured
                               // 36 % slower on corpus200 (spills, no IN(dst) pre-read): off
#endif
#ifndef GD_CONT_WIDE
#define GD_CONT_WIDE 1         // wide items continue depth-first into wide successors
#endif
#ifndef GD_CONT_DENSE
#define GD_CONT_DENSE 1        // continue into narrow (one word per row) destinations too (light rounds)
#endif
constexpr uint32_t NO_CONT = 0xffffffffu;
constexpr uint32_t ROUND_SWITCH = 0xffffffffu;   // run_round: leave this launch before the round

struct Acc {                   // per-warp counters (shared memory), flushed once per kernel
  unsigned long long alg;      // touched-word model bytes
  unsigned long long dense;    // dense-model bytes
  unsigned long long atom;     // RED.OR issued
  unsigned long long cont;     // items processed by continuation (visits not in the queue)
};

template <bool WIDE>
struct WarpScratchT {
  uint64_t rv[MAXW];           // FSTORE base row v
  uint64_t rw[MAXW];           // FSTORE / FLOAD value row w
  uint64_t gen[MAXW];          // generated row (wide path)
  int16_t cmap[64 * MAXW];     // projection column map of the current cross-module edge
  uint16_t rowlist[WIDE ? 1024 : 1];        // wide: candidate rows, then the rows with OUT_Δ != 0
  uint32_t gbits[WIDE ? 32 : 1];            // wide: update() per edge of the item (<= 1024 edges)
};

// warp-uniform counter updates: lane 0 adds the warp's total
__device__ __forceinline__ void acc_add(unsigned long long& slot, uint32_t per_lane) {
  const uint32_t t = __reduce_add_sync(FULL, per_lane);
  if ((threadIdx.x & 31) == 0) slot += t;
}

struct CtaStage {              // per-CTA staged worklist appends of the current round
  uint32_t cnt[NCLS];
  uint32_t nodes;
  uint32_t gbase[NCLS];
  uint32_t buf[NCLS][SCAP];
  // SBDA schedule (k_sbda): the CTA's method-local worklists in shared memory
  uint32_t* lq;                // [2][LQCAP] entries (node << 5 | chunk), LQ_SKIP = empty slot
  uint32_t lcnt[2];
  uint32_t lsel;               // local queue being processed
  unsigned long long lid;      // local round id (pass << 32 | counter): dedupe key in D.lstamp
};
constexpr uint32_t LQCAP = 1024;
#ifndef GD_CONT_STAMP
#define GD_CONT_STAMP 1
#endif
#ifndef GD_DYN
#define GD_DYN 1             // wide batches: dynamic item hand-out within a round (run_round)
#endif
#ifndef GD_DIG_U2
#define GD_DIG_U2 0          // k_digest: two bits of a word per loop iteration (A/B: +0.3 %, off)
#endif
#ifndef GD_DIG2
#define GD_DIG2 0            // k_digest: bits spread over the lanes (digest_words2; A/B: corpus +8.8 %, off)
#endif
#ifndef GD_ITEM3
#define GD_ITEM3 1           // non-inline narrow items of blocks <= 96 words: 3 words per lane
#endif
#ifndef GD_INL4
#define GD_INL4 1            // inline path for blocks of 97..128 words too (4 words per lane)
#endif
#ifndef GD_INL2
#define GD_INL2 0            // inline items of blocks <= 64 words: 2 words per lane (A/B: corpus +5.7 %, off)
#endif
#ifndef GD_INL3
#define GD_INL3 1            // inline items of blocks <= 96 words: 3 words per lane instead of 4
#endif
#ifndef GD_DYN_NARROW
#define GD_DYN_NARROW 0      // narrow batches too (A/B)
#endif
#ifndef GD_DYN_GRAIN
#define GD_DYN_GRAIN 8       // narrow batches: items per claim
#endif
#ifndef GD_CONT_PF
#define GD_CONT_PF 0         // light rounds: prefetch the inline successors' records into L1 (A/B: small +6 %, off)
#endif
constexpr uint32_t LQ_SKIP = 0xffffffffu;

// fire-and-forget 64-bit OR at L2 (RED; no return value, no scoreboard wait)
__device__ __forceinline__ void red_or(uint64_t* p, uint64_t v) {
  asm volatile("red.relaxed.gpu.global.or.b64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

// Narrow word-occupancy masks (GD_NMASK): bit w of the node's 2 mask words = word w of IN(n) may
// be non-zero (words >= 128 are never masked).  A writer that turns a word non-zero sets the bit
// (one RED, at most once per word per build in practice); a reader that misses a bit still in
// flight is re-run next round, because that writer also queued the node.
__device__ __forceinline__ void nmask_note(uint64_t* m, uint32_t w) {
  if (GD_NMASK && w < 64u * NMW) red_or(m + (w >> 6), 1ull << (w & 63));
}
__device__ __forceinline__ bool nmask_has(uint64_t m0, uint64_t m1, uint32_t w) {
  return !GD_NMASK || w >= 64u * NMW || (((w < 64 ? m0 : m1) >> (w & 63)) & 1ull);
}

// fire-and-forget 64-bit AND at L2 (clears the Δ bits a visit consumed)
__device__ __forceinline__ void red_and(uint64_t* p, uint64_t v) {
  asm volatile("red.relaxed.gpu.global.and.b64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t warp_or64(uint64_t v) {
  const uint32_t lo = __reduce_or_sync(FULL, (uint32_t)v);
  const uint32_t hi = __reduce_or_sync(FULL, (uint32_t)(v >> 32));
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

// ---------------------------------------------------------------------------------- pushes
__device__ __forceinline__ void stage_init(CtaStage& st) {
  if (threadIdx.x < NCLS) st.cnt[threadIdx.x] = 0;
  if (threadIdx.x == NCLS) st.nodes = 0;
}

// Append the candidate destinations held by the warp's lanes (every chunk of a pushed node)
// to the CTA's staged worklist of the next round.
//
// Continuation (cont != nullptr, warp-uniform *cont == NO_CONT on entry): the first lane whose
// single-chunk destination (not queued for this round or the next) wants a visit may instead hand it back to the
// warp, which processes it at once in this round (a depth-first step).  That lane
// does not queue it: the warp reads IN(dst) after its own ORs, and a later grower of dst sees a
// stamp below round+1 and queues dst as usual, so no growth is lost.  The claim is one
// atomicMax(stamp[dst], round) returning a value below round: it keeps a second warp from
// continuing into the same node in the same round (it queues it instead) and a node already
// queued for this round or the next from being continued into (GD_CONT_STAMP; the round-2 claim
// was a stamp load, an atomicExch on cont[dst] and the atomicMax: three dependent L2 hops).
template <bool SB = false>
__device__ __forceinline__ void flush_pushes(const Dev& D, CtaStage& st, int lane, bool active,
                                             uint32_t dst, uint32_t info, bool grew, uint32_t round,
                                             uint32_t nxt, uint32_t* cont = nullptr, bool cont_dense = false,
                                             uint32_t pre_stamp = NO_CONT) {
  bool push = false;
  bool want = false;
  // grew, or first reach (A5).  pre_stamp: stamp[dst] loaded early by the caller (a stale value
  // is safe: stamps only grow, and the atomicMax below decides the push)
  uint32_t sv = 0;
  if (active) {
    sv = pre_stamp != NO_CONT ? pre_stamp : D.stamp[dst];
    want = grew || sv == 0;
  }
  if constexpr (SB) {
    // SBDA: an INTRA / C2R successor belongs to the method this CTA is solving,
    // so it joins the CTA's next local round (deduplicated per local round through D.lstamp);
    // CALL / RET successors go to the next pass through the global worklist below.
    const uint32_t ek = info & 3u;
    if (want && (ek == GE_INTRA || ek == GE_C2R)) {
      atomicMax(&D.stamp[dst], round);                     // reached (first-reach history)
      const unsigned long long lid = st.lid;
      if (atomicMax((unsigned long long*)&D.lstamp[dst], lid) < lid) {
        const uint32_t nch = ((info >> 5) & 31u) + 1, nl = st.lsel ^ 1u;
        const uint32_t base = atomicAdd(&st.lcnt[nl], nch);
        if (base + nch <= LQCAP) {
          for (uint32_t q = 0; q < nch; ++q) st.lq[nl * LQCAP + base + q] = (dst << 5) | q;
          want = false;
        } else {                                            // local queue full: next pass
          for (uint32_t q = base; q < LQCAP; ++q) st.lq[nl * LQCAP + q] = LQ_SKIP;
        }
      } else {
        want = false;                                      // already in the next local round
      }
    }
  }
  bool decided = false;                                     // pushes already decided below
  if (cont && *cont == NO_CONT && (D.flags & F_CONT)) {
#if GD_CONT_STAMP
    // One memory hop for every wanting lane: the candidate claims the continuation with
    // atomicMax(stamp[dst], round) — below round before: not queued for this round or the next,
    // not continued into by another warp this round — while the other lanes queue theirs for the
    // next round (stamp -> round + 1) with the same instruction.  The stamp loaded with the item's
    // first hop (sv, possibly stale: stamps only grow) picks the candidate.
    const unsigned cand = __ballot_sync(FULL, want && sv < round && (cont_dense || (info & INFO_WIDE)) &&
                                                  ((info >> 5) & 31u) == 0);
    const int l = cand ? __ffs(cand) - 1 : -1;
    const bool issue = active && want && (lane == l || sv != round + 1);
    uint32_t old = 0;
    if (issue) old = atomicMax(&D.stamp[dst], lane == l ? round : round + 1);
    uint32_t ok = 0;
    if (lane == l) {
      if (old < round) { ok = 1; want = false; }
      else if (old == round) push = atomicMax(&D.stamp[dst], round + 1) < round + 1;   // rare: queue it
    } else if (issue) {
      push = old < round + 1;
    }
    decided = true;
    if (l >= 0 && __shfl_sync(FULL, ok, l)) *cont = __shfl_sync(FULL, dst, l);
#else
    const unsigned cand = __ballot_sync(FULL, want && (cont_dense || (info & INFO_WIDE)) && ((info >> 5) & 31u) == 0);
    if (cand) {
      const int l = __ffs(cand) - 1;
      uint32_t ok = 0;
      if (lane == l && D.stamp[dst] < round && atomicExch(&D.cont[dst], round) != round) {
        atomicMax(&D.stamp[dst], round);                    // reached: no first-reach pushes
        ok = 1;
        want = false;
      }
      if (__shfl_sync(FULL, ok, l)) *cont = __shfl_sync(FULL, dst, l);
    }
#endif
  }
  if (active && !decided) {
    // sv == round + 1: already queued for the next round (stamps never exceed round + 1 during
    // round `round`, and a stale value is never larger than the true one) — no atomic needed
    if (want && sv != round + 1) {
      const uint32_t old = atomicMax(&D.stamp[dst], round + 1);  // test-and-set: de-duplicates (MER)
      push = old < round + 1;
    }
  }
  const int cls = push ? ((D.flags & F_GRP) ? (int)((info >> 2) & 7u) : 0) : -1;   // GRP segment
  const uint32_t nch = ((info >> 5) & 31u) + 1;
  unsigned pm = __ballot_sync(FULL, push);
  if (__popc(pm) == 1) {                                     // common case: one destination
    if (push) {
      atomicAdd(&st.nodes, 1u);
      const uint32_t base = atomicAdd(&st.cnt[cls], nch);
      for (uint32_t q = 0; q < nch; ++q) {
        const uint32_t idx = base + q, entry = (dst << 5) | q;
        if (idx < (uint32_t)SCAP) st.buf[cls][idx] = entry;
        else {
          const uint32_t g = atomicAdd(&D.counts[nxt * CNT_STRIDE + cls], 1u);
          D.queue[(size_t)nxt * D.n_chunks + D.seg[cls] + g] = entry;
        }
      }
    }
    return;
  }
  if (pm && lane == 0) atomicAdd(&st.nodes, (uint32_t)__popc(pm));
  while (pm) {                                               // warp-aggregated append per class
    const int leader = __ffs(pm) - 1;
    const int c = __shfl_sync(FULL, cls, leader);
    const bool mine = push && cls == c;
    const unsigned same = __ballot_sync(FULL, mine);
    const uint32_t v = mine ? nch : 0u;
    uint32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(FULL, incl, o);
      if (lane >= o) incl += t;
    }
    const uint32_t total = __shfl_sync(FULL, incl, 31);
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(&st.cnt[c], total);
    base = __shfl_sync(FULL, base, leader);
    if (mine) {
      for (uint32_t q = 0; q < nch; ++q) {
        const uint32_t idx = base + (incl - v) + q;
        const uint32_t entry = (dst << 5) | q;
        if (idx < (uint32_t)SCAP) st.buf[c][idx] = entry;
        else {                                                 // stage full: publish directly
          const uint32_t g = atomicAdd(&D.counts[nxt * CNT_STRIDE + c], 1u);
          D.queue[(size_t)nxt * D.n_chunks + D.seg[c] + g] = entry;
        }
      }
    }
    pm &= ~same;
  }
}

// Publish the CTA's staged appends (one global atomic per class), then reset the stage.
__device__ __forceinline__ void stage_publish(const Dev& D, CtaStage& st, uint32_t nxt) {
  __syncthreads();
  if (threadIdx.x < NCLS) {
    const uint32_t n = min(st.cnt[threadIdx.x], (uint32_t)SCAP);
    st.gbase[threadIdx.x] = n ? atomicAdd(&D.counts[nxt * CNT_STRIDE + threadIdx.x], n) : 0u;
  }
  if (threadIdx.x == NCLS && st.nodes) atomicAdd(&D.counts[nxt * CNT_STRIDE + CNT_NODES], st.nodes);
  __syncthreads();
#pragma unroll
  for (int c = 0; c < NCLS; ++c) {
    const uint32_t n = min(st.cnt[c], (uint32_t)SCAP);
    uint32_t* q = D.queue + (size_t)nxt * D.n_chunks + D.seg[c] + st.gbase[c];
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) q[i] = st.buf[c][i];
  }
  __syncthreads();
  stage_init(st);
}

// ---------------------------------------------------------------------------------- unions
// OR KW words into IN(dst): a (possibly stale) load, then RED.OR only where bits are missing.
// Words of row `kill` are dropped (C2R).  Returns the number of non-zero words in the low
// 16 bits and the number of REDs issued in the high bits.
template <int K>
__device__ __forceinline__ uint32_t or_chunk(uint64_t* Z, const uint64_t (&y)[K], uint32_t c0,
                                             int lane, int kill, uint32_t logW, uint64_t* zm) {
  uint64_t cur[K];
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint32_t w = c0 + lane + 32 * k;
    const bool keep = y[k] && !(kill >= 0 && (int)(w >> logW) == kill);
    cur[k] = keep ? Z[w] : ~0ull;
  }
  uint32_t nz = 0, red = 0;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint32_t w = c0 + lane + 32 * k;
    const uint64_t z = (kill >= 0 && (int)(w >> logW) == kill) ? 0ull : y[k];
    nz += (z != 0);
    if (z & ~cur[k]) {
      red_or(Z + w, z);
      ++red;
      if (cur[k] == 0) nmask_note(zm, w);                         // zero word becomes non-zero
    }
  }
  return nz | (red << 16);
}


// ---------------------------------------------------------------------------------- wide blocks
// Row-sparse processing of a node whose block is wide (W >= 2 words per row): only the rows
// flagged in its occupancy bitmap (plus the rows its transfer function generates) are read,
// transformed and propagated; every row written into a wide target also sets the target's
// occupancy bit.  Same results as the dense path, bytes proportional to non-zero rows.
constexpr int WROWS = 1024;    // row-list capacity per warp (rows of one block)

// OR one row into IN(dst) (wide or narrow target).  Wide targets (logWt >= 1) also get the
// new bits in Δ(dst) (Zd: the target's block in the Δ store), which their next visit consumes.
template <int MW>
__device__ __forceinline__ void emit_row_words(uint64_t* Z, uint32_t Bt, uint32_t logWt, uint32_t rt,
                                               const uint64_t (&v)[MW], uint32_t& nz, uint32_t& red, bool& g,
                                               uint64_t* mask_t, uint64_t* Zd) {
  const uint32_t Wt = 1u << logWt;
  uint64_t* row = Z + ((uint64_t)rt << logWt);
  uint64_t cur[MW];
  bool any = false, was_zero = true;
#pragma unroll
  for (int j = 0; j < MW; ++j) {
    cur[j] = (j < (int)Wt && v[j]) ? row[j] : ~0ull;
    any |= (j < (int)Wt && v[j] != 0);
  }
  if (!any) return;
  bool wrote = false;
#pragma unroll
  for (int j = 0; j < MW; ++j) {
    if (j >= (int)Wt || !v[j]) continue;
    ++nz;
    if (cur[j]) was_zero = false;
    const uint64_t nb = v[j] & ~cur[j];
    if (nb) {
      red_or(row + j, v[j]);
      if (logWt >= 1) red_or(Zd + ((uint64_t)rt << logWt) + j, nb);   // Δ(dst) of a wide target
      ++red; g = true; wrote = true;
    }
  }
  if (logWt >= 1 && was_zero) red_or(Z + occ_offset(Bt) + (rt >> 6), 1ull << (rt & 63));   // occupancy
  if (logWt == 0 && was_zero && wrote) nmask_note(mask_t, rt);   // narrow target: word-occupancy
}

// Semi-naive (Δ) visit of a wide block.  IN(src) supplies the transfer
// function's operand rows and the candidate rows (its row-occupancy bitmap); the visit
// propagates only OUT_Δ = (Δ(src) \ KILL) ∪ GEN(IN(src)) where Δ(src) holds the bits that
// reached IN(src) since its last visit.  Every f of §3 C2 is (X \ KILL) ∪ GEN(X) with GEN
// monotone and every edge transform distributes over ∪, so f(IN_old ∪ Δ) ⊆ f(IN_old) ∪ OUT_Δ:
// successors already hold T_e(f(IN_old)) from earlier visits and receive T_e(OUT_Δ) now —
// the same least fixed point (C4) with work proportional to the new facts.  Δ bits are
// consumed with RED.AND of exactly the bits read; bits arriving later stay for the next visit
// (their writer also queued the node).
template <bool CNT, int MW, bool SB = false>
__device__ void process_wide(const Dev& D, CtaStage& st, const NodeRec& R, uint32_t n, uint32_t e0, uint32_t e1,
                             bool first, uint32_t round, uint32_t nxt, int lane, WarpScratchT<true>& ws, Acc& acc,
                             uint32_t alg_l0, uint32_t* cont, bool cont_dense) {
  const uint32_t logW = R.logW, W = 1u << logW, L = R.L, B = R.B, rows = B >> logW;
  // The fact store is read and RED.OR-ed by the same kernel (self loops write IN(src) within
  // one item): no __restrict__ / const-cache loads on it, only plain coherent LDG.
  const uint64_t* X = D.facts + R.off;
  uint64_t* DX = D.delta + R.off;
  const uint64_t* OCC = X + occ_offset(B);
  const uint32_t nocc = occ_words(rows);
  const uint32_t kind = R.kind;
  if (lane < (int)min(e1 - e0, 32u))                       // edge records into L1 (read in pass 2)
    asm volatile("prefetch.global.L1 [%0];" :: "l"((const char*)(D.edges + e0 + lane)));
  // ---- transfer setup on IN(src): generated row t (mode 1 replace / 2 or-in) or FSTORE rows
  //      (mode 3).  The full GEN is emitted on every visit (a superset of its new part).
  int mode = 0, t = -1;
  uint32_t hwords = 0;
  if (lane < MAXW) ws.gen[lane] = 0;
  if (kind == GK_PRIM || kind == GK_CONST || kind == GK_NEW) {
    mode = 1; t = R.r0;
    if (kind != GK_PRIM && lane == (R.r3 >> 6)) ws.gen[lane] = 1ull << (R.r3 & 63);
  } else if (kind == GK_COPY || kind == GK_SLOAD || kind == GK_RETV || kind == GK_SSTORE) {
    mode = kind == GK_SSTORE ? 2 : 1; t = R.r0;
    if (lane < (int)W) ws.gen[lane] = X[((uint64_t)R.r1 << logW) + lane];
  } else if (kind == GK_FLOAD || kind == GK_ALOAD) {
    mode = 1; t = R.r0;
    if (lane < (int)W) ws.rw[lane] = X[((uint64_t)R.r1 << logW) + lane];
    __syncwarp();
    uint64_t a[MW];
#pragma unroll
    for (int j = 0; j < MW; ++j) a[j] = 0;
    for (uint32_t c = lane; c < R.n_cols; c += 32) {
      if (!((ws.rw[c >> 6] >> (c & 63)) & 1ull)) continue;
      const int hr = D.frow[R.r3 + c];
      if (hr < 0) continue;                                  // NULL / field not declared
      const uint64_t* H = X + ((uint64_t)(L + hr) << logW);
#pragma unroll
      for (int j = 0; j < MW; ++j)
        if (j < (int)W) a[j] |= H[j];
      hwords += W;
    }
#pragma unroll
    for (int j = 0; j < MW; ++j)
      if (j < (int)W) {
        const uint64_t v = warp_or64(a[j]);
        if (lane == j) ws.gen[j] = v;
      }
  } else if (kind == GK_FSTORE || kind == GK_ASTORE) {
    mode = 3;
    if (lane < (int)W) {
      ws.rv[lane] = X[((uint64_t)R.r0 << logW) + lane];
      ws.rw[lane] = X[((uint64_t)R.r1 << logW) + lane];
    }
  }
  if (lane < 32) ws.gbits[lane] = 0;
  __syncwarp();
  // ---- candidate rows: IN-occupied rows (Δ ⊆ IN), then generated rows not occupied yet
  const unsigned lt_mask = (1u << lane) - 1u;
  const uint64_t my_occ = lane < (int)nocc ? OCC[lane] : 0ull;   // nocc <= 32 (loader: rows <= WROWS)
  uint32_t cnt = 0;
  for (uint32_t i = 0; i < nocc; ++i) {
    const uint64_t wv = __shfl_sync(FULL, my_occ, i);
    const uint32_t lo = (uint32_t)wv, hi = (uint32_t)(wv >> 32);
    if ((lo >> lane) & 1u) ws.rowlist[cnt + __popc(lo & lt_mask)] = (uint16_t)(i * 64 + lane);
    if ((hi >> lane) & 1u) ws.rowlist[cnt + __popc(lo) + __popc(hi & lt_mask)] = (uint16_t)(i * 64 + 32 + lane);
    cnt += __popc(lo) + __popc(hi);
  }
  if (mode == 1 || mode == 2) {
    const uint64_t wv = __shfl_sync(FULL, my_occ, (uint32_t)t >> 6);
    if (!((wv >> (t & 63)) & 1ull)) { if (lane == 0) ws.rowlist[cnt] = (uint16_t)t; ++cnt; }
  } else if (mode == 3) {                                    // heap rows (o1, f), o1 in row v
    for (uint32_t c0 = 0; c0 < R.n_cols; c0 += 32) {
      const uint32_t c = c0 + lane;
      int hr = -1;
      if (c < R.n_cols && ((ws.rv[c >> 6] >> (c & 63)) & 1ull)) hr = D.frow[R.r3 + c];
      const uint32_t r = hr >= 0 ? L + (uint32_t)hr : 0u;
      const uint64_t wv = __shfl_sync(FULL, my_occ, r >> 6);
      const bool need = hr >= 0 && !((wv >> (r & 63)) & 1ull);
      const unsigned m = __ballot_sync(FULL, need);
      if (need) ws.rowlist[cnt + __popc(m & lt_mask)] = (uint16_t)r;
      cnt += __popc(m);
    }
  }
  __syncwarp();

  uint32_t nzx = 0, nz = 0, red = 0;
  unsigned long long dense_l0 = first ? 8ull * B : 0ull;
  // OUT_Δ row of candidate row r: Δ(src) row r (killed for mode-1 row t), plus the GEN rows
  auto out_delta = [&](uint32_t r, uint64_t (&y)[MW], bool consume) {
    uint64_t* drow = DX + ((uint64_t)r << logW);
#pragma unroll
    for (int j = 0; j < MW; ++j) y[j] = (j < (int)W) ? drow[j] : 0ull;
    if (consume) {
#pragma unroll
      for (int j = 0; j < MW; ++j)
        if (y[j]) { red_and(drow + j, ~y[j]); ++nzx; }      // consume exactly the bits read
    }
    if (mode == 1 && (int)r == t) {                          // Δ row t killed, GEN instead
#pragma unroll
      for (int j = 0; j < MW; ++j) y[j] = (j < (int)W) ? ws.gen[j] : 0ull;
    } else if (mode == 2 && (int)r == t) {
#pragma unroll
      for (int j = 0; j < MW; ++j) if (j < (int)W) y[j] |= ws.gen[j];
    } else if (mode == 3 && r >= L + R.n_stat) {
      const uint32_t gg = r - L;
      if (D.grow_field[R.grow_off + gg] == R.r2) {
        const int c = D.grow_col[R.grow_off + gg];
        if ((ws.rv[c >> 6] >> (c & 63)) & 1ull) {
#pragma unroll
          for (int j = 0; j < MW; ++j) if (j < (int)W) y[j] |= ws.rw[j];
        }
      }
    }
    bool any = false;
#pragma unroll
    for (int j = 0; j < MW; ++j) any |= (y[j] != 0);
    return any;
  };
  // ---- pass 1: keep the candidate rows whose OUT_Δ is non-empty (compacted in place; a row
  //      that gains Δ bits after this scan keeps them for the node's next visit)
  //      (at most 32 candidates: no compaction, pass 2 reads every candidate once)
  uint32_t kept = cnt <= 32 ? cnt : 0u;
  for (uint32_t p0 = 0; cnt > 32 && p0 < cnt; p0 += 32) {
    const uint32_t p = p0 + lane;
    uint64_t y[MW];
    const uint32_t r = p < cnt ? ws.rowlist[p] : 0u;
    const bool keep = p < cnt && out_delta(r, y, false);
    const unsigned km = __ballot_sync(FULL, keep);
    if (keep) ws.rowlist[kept + __popc(km & lt_mask)] = (uint16_t)r;   // (behind every read)
    kept += __popc(km);
  }
  __syncwarp();
  // ---- pass 2: 32 kept rows at a time (one per lane): consume their Δ bits and propagate
  //      OUT_Δ along every edge of the item
  for (uint32_t q0 = 0; q0 < kept; q0 += 32) {
    const bool mine = q0 + lane < kept;
    const uint32_t rr = mine ? ws.rowlist[q0 + lane] : 0u;
    uint64_t yv[MW];
    const bool live = mine && out_delta(rr, yv, true);
    for (uint32_t e = e0; e < e1; ++e) {
      const Edge* ep = D.edges + e;
      const uint32_t ek = ep->info & 3u;
      uint64_t* Z = D.facts + ep->off;
      uint64_t* Zd = D.delta + ep->off;
      const uint32_t Bt = ep->B, Lt = ep->L, logWt = ep->logW;
      const int aux = ep->aux;
      const uint32_t xoff = ep->xoff;
      const bool proj = (ek == GE_CALL || ek == GE_RET) && xoff != NO_XMAP;
      if (proj) {
        for (uint32_t c = lane; c < R.n_cols; c += 32) ws.cmap[c] = (int16_t)D.xmap[xoff + c];
        __syncwarp();
      }
      const int32_t* rowinv = proj ? D.xmap + xoff + R.n_cols + ((Bt >> logWt) - Lt) : nullptr;
      const uint32_t npar = (ek == GE_CALL) ? (uint32_t)aux : 0u;
      const int lhs = (ek == GE_RET) ? aux : -1;
      bool g = false;
      if (live) {
        // Target rows.  Every edge kind maps source row rr to at most one target row, except
        // CALL locals: one local passed as several actuals feeds every such parameter
        // (param_j <- arg_j for all j), so CALL scans all npar actuals.
        int rt = -1;
        const bool call_local = ek == GE_CALL && rr < L;
        if (ek == GE_INTRA) rt = (int)rr;
        else if (ek == GE_C2R) rt = ((int)rr == R.r0) ? -1 : (int)rr;
        else if (rr >= L) {
          const uint32_t gs = rr - L;
          const int gt = proj ? rowinv[gs] : (int)gs;       // π: source global row -> target row
          if (gt >= 0) rt = (int)Lt + gt;
        } else if (ek == GE_RET) {
          if (rr == L - 1 && lhs >= 0) rt = lhs;
        }
        if (rt >= 0 || call_local) {
          uint64_t out[MW];                                 // the row in the target's columns
          if (!proj) {
#pragma unroll
            for (int s2 = 0; s2 < MW; ++s2) out[s2] = yv[s2];
          } else {
#pragma unroll
            for (int s2 = 0; s2 < MW; ++s2) out[s2] = 0;
            for (uint32_t j = 0; j < W; ++j) {
              uint64_t b = 0;
#pragma unroll
              for (int jj = 0; jj < MW; ++jj) if ((uint32_t)jj == j) b = yv[jj];
              while (b) {
                const int bit = __ffsll((long long)b) - 1;
                b &= b - 1;
                const int cd = ws.cmap[j * 64 + bit];
                if (cd < 0) continue;
#pragma unroll
                for (int s2 = 0; s2 < MW; ++s2)
                  if (s2 == (cd >> 6)) out[s2] |= 1ull << (cd & 63);
              }
            }
          }
          if (!call_local) {
            emit_row_words(Z, Bt, logWt, (uint32_t)rt, out, nz, red, g, D.smask + (uint64_t)NMW * ep->dst, Zd);
          } else {
            const uint32_t a0 = npar > 3 ? D.arg_ptr[n] : 0u;
            for (uint32_t jj = 0; jj < npar; ++jj) {        // param_jj <- arg_jj whenever arg_jj = rr
              const int a = npar > 3 ? D.args[a0 + jj] : (jj == 0 ? R.r1 : (jj == 1 ? R.r2 : R.r3));
              if (a == (int)rr) emit_row_words(Z, Bt, logWt, jj, out, nz, red, g, D.smask + (uint64_t)NMW * ep->dst, Zd);
            }
          }
        }
      }
      if (proj) __syncwarp();
      if (__any_sync(FULL, g) && lane == 0 && e - e0 < 1024u) ws.gbits[(e - e0) >> 5] |= 1u << ((e - e0) & 31u);
      if (q0 == 0) dense_l0 += 16ull * Bt;
    }
  }
  __syncwarp();
  for (uint32_t eb = e0; eb < e1; eb += 32) {               // update() / first reach -> pushes
    const uint32_t ne = min(32u, e1 - eb);
    const uint32_t gm = eb - e0 < 1024u ? ws.gbits[(eb - e0) >> 5] : ~0u;   // beyond: push (safe)
    const uint32_t my_info = lane < (int)ne ? D.edges[eb + lane].info : 0u;
    const uint32_t my_dst = lane < (int)ne ? D.edges[eb + lane].dst : 0u;
    flush_pushes<SB>(D, st, lane, lane < (int)ne, my_dst, my_info, (gm >> lane) & 1u, round, nxt, cont, cont_dense);
  }
  if constexpr (CNT) {                     // byte models (dead code, removed, when !CNT)
    // touched words of the semi-naive visit: Δ(src) words read and cleared, T_e(OUT_Δ) words
    // read and OR-ed into IN(dst) (+ Δ(dst)), heap rows gathered, occupancy words
    acc_add(acc.alg, 24u * nz + 16u * nzx + 8u * hwords + 8u * nocc + (lane == 0 ? alg_l0 : 0u));
    acc_add(acc.atom, red);
    if (lane == 0) acc.dense += dense_l0 + alg_l0;
  }
}

// ---------------------------------------------------------------------------------- inline items
__device__ __forceinline__ uint64_t hshfl_xor64(uint64_t v, int o) {   // xor within the half-warp
  const uint32_t lo = __shfl_xor_sync(FULL, (uint32_t)v, o, 16), hi = __shfl_xor_sync(FULL, (uint32_t)(v >> 32), o, 16);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
  const uint32_t lo = __shfl_sync(FULL, (uint32_t)v, src), hi = __shfl_sync(FULL, (uint32_t)(v >> 32), src);
  return ((uint64_t)hi << 32) | lo;
}
// Word r of a block held as y[k] = word lane + 32k.  uword_of: r warp-uniform (one shuffle);
// word_of: r per lane (every lane takes part).
template <int K>
__device__ __forceinline__ uint64_t uword_of(const uint64_t (&y)[K], uint32_t r) {
  uint64_t s = y[0];
#pragma unroll
  for (int k = 1; k < K; ++k) if ((r >> 5) == (uint32_t)k) s = y[k];
  return shfl64(s, (int)(r & 31u));
}
template <int K>
__device__ __forceinline__ uint64_t word_of(const uint64_t (&y)[K], uint32_t r) {
  uint64_t s = 0;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint64_t v = shfl64(y[k], (int)(r & 31u));
    if ((r >> 5) == (uint32_t)k) s = v;
  }
  return s;
}

// Chunk 0 of a narrow node (block of <= 128 words) whose edges are all INTRA/C2R and held in
// the node's inline record (NodeRec::n_inl).  Same transfer and union as process_item's narrow
// path, with every read that the chain allows issued in the first memory hop: IN(src), the
// destinations' round stamps and (FLOAD/FSTORE) the field-row table; the rows the transfer
// function reads are taken from the IN(src) registers by shuffles instead of reloads.
template <bool CNT, bool CD, bool SB = false, int K = KW>
__device__ __forceinline__ uint32_t process_inline(const Dev& D, CtaStage& st, const NodeRec& R, const InlEdge& me,
                                                   uint32_t round, uint32_t nxt, int lane, Acc& acc,
                                                   bool cont_ok, uint64_t mk0, uint64_t mk1) {
  const uint32_t B = R.B, L = R.L, ne = R.n_inl, kind = R.kind;
  const uint64_t* X = D.facts + R.off;             // coherent loads (no __restrict__: see process_wide)
  uint64_t y[K], p0[K], p1[K];
  const uint64_t off0 = shfl64(me.off, 0), off1 = shfl64(me.off, 1);
  uint32_t hasm = 0;                                        // bit k: word lane + 32k may be non-zero
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint32_t w = lane + 32 * k;
    const bool h = w < B && nmask_has(mk0, mk1, w);
    hasm |= (uint32_t)h << k;
    y[k] = h ? X[w] : 0ull;
    if (GD_PRE) {                                           // IN(dst) of edges 0 and 1, same hop
      p0[k] = h ? D.facts[off0 + w] : 0ull;                 // (only words IN(src) may carry)
      if (GD_PRE2) p1[k] = (ne > 1 && h) ? D.facts[off1 + w] : 0ull;
    }
  }
  const uint32_t my_stamp = lane < (int)ne ? D.stamp[me.dst] : 1u;
  if (GD_CONT_PF && CD && cont_ok && lane < (int)ne) {       // a continuation's first hop hits L1
    asm volatile("prefetch.global.L1 [%0];" :: "l"((const char*)(D.nodes + me.dst)));
    asm volatile("prefetch.global.L1 [%0];" :: "l"((const char*)(D.inl + 4 * me.dst)));
  }
  const bool dbl = kind == GK_FLOAD || kind == GK_ALOAD || kind == GK_FSTORE || kind == GK_ASTORE;
  int hr[2] = {-1, -1};                                     // heap rows of this lane's columns
  if (dbl) {
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const uint32_t c = lane + 32 * q;
      hr[q] = (c < R.n_cols) ? D.frow[R.r3 + c] : -1;
    }
  }
  // ---- transfer (DESIGN.md §3 C2), on the registers
  int mode = 0, t = -1;                                     // 0 identity, 1 replace, 2 or-in, 3 FSTORE
  uint64_t genv = 0;
  uint32_t fmask = 0, hwords = 0;
  if (kind == GK_PRIM || kind == GK_CONST || kind == GK_NEW) {
    mode = 1; t = R.r0;
    if (kind != GK_PRIM) genv = 1ull << (R.r3 & 63);
  } else if (kind == GK_COPY || kind == GK_SLOAD || kind == GK_RETV || kind == GK_SSTORE) {
    mode = kind == GK_SSTORE ? 2 : 1; t = R.r0;
    genv = uword_of(y, (uint32_t)R.r1);                     // row rhs
  } else if (kind == GK_FLOAD || kind == GK_ALOAD) {       // v = w.f: OR of rows (o1,f), o1 ∈ w
    mode = 1; t = R.r0;
    const uint64_t wrow = uword_of(y, (uint32_t)R.r1);
    uint64_t a = 0;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const uint32_t c = lane + 32 * q;
      const bool take = hr[q] >= 0 && ((wrow >> c) & 1ull);  // NULL has no row
      const uint64_t v = word_of(y, take ? L + (uint32_t)hr[q] : 0u);
      if (take) { a |= v; hwords += 1; }
    }
    genv = warp_or64(a);
  } else if (kind == GK_FSTORE || kind == GK_ASTORE) {     // v.f = w (weak)
    mode = 3;
    const uint64_t vrow = uword_of(y, (uint32_t)R.r0);
    genv = uword_of(y, (uint32_t)R.r1);                     // row w, OR-ed into rows (o1, f)
#pragma unroll
    for (int k = 0; k < K; ++k) {
      uint32_t m = 0;
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const uint32_t c = lane + 32 * q;
        if (hr[q] >= 0 && ((vrow >> c) & 1ull)) {
          const uint32_t w = L + (uint32_t)hr[q];
          if ((w >> 5) == (uint32_t)k) m |= 1u << (w & 31u);
        }
      }
      m = __reduce_or_sync(FULL, m);
      if ((m >> lane) & 1u) fmask |= 1u << k;
    }
  }
  uint32_t nzx = 0, nz = 0, red = 0;
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint32_t w = lane + 32 * k;
    if (CNT) nzx += (y[k] != 0);
    if (mode == 1) { if ((int)w == t) y[k] = genv; }
    else if (mode == 2) { if ((int)w == t) y[k] |= genv; }
    else if (mode == 3) { if ((fmask >> k) & 1u) y[k] |= genv; }
  }
  // ---- unions into IN(dst) (a5)
  unsigned gmask = 0;
  for (uint32_t i = 0; i < ne; ++i) {
    const uint64_t off = shfl64(me.off, (int)i);
    const uint32_t info = __shfl_sync(FULL, me.info, (int)i);
    const int kill = ((info & 3u) == GE_C2R) ? R.r0 : -1;  // C2R drops lhs(c)
    uint64_t* Z = D.facts + off;
    uint64_t* zm = D.smask + (uint64_t)NMW * __shfl_sync(FULL, me.dst, (int)i);
    uint64_t cur[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t w = lane + 32 * k;
      const bool keep = y[k] && (int)w != kill;
      const bool pre = (hasm >> k) & 1u;                    // pre-read done for this word
      if (GD_PRE && i == 0) cur[k] = keep ? (pre ? p0[k] : Z[w]) : ~0ull;
      else if (GD_PRE && GD_PRE2 && i == 1) cur[k] = keep ? (pre ? p1[k] : Z[w]) : ~0ull;
      else cur[k] = keep ? Z[w] : ~0ull;
    }
    bool g = false;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t w = lane + 32 * k;
      const uint64_t z = (int)w == kill ? 0ull : y[k];
      nz += (z != 0);
      if (z & ~cur[k]) {
        red_or(Z + w, z); ++red; g = true;
        if (cur[k] == 0) nmask_note(zm, w);                 // zero word becomes non-zero
      }
    }
    if (__any_sync(FULL, g)) gmask |= 1u << i;
  }
  uint32_t cont_v = NO_CONT;                               // GD_CONT_DENSE: depth-first successor
  flush_pushes<SB>(D, st, lane, lane < (int)ne, me.dst, me.info, (gmask >> lane) & 1u, round, nxt,
               (CD && cont_ok) ? &cont_v : nullptr, true, my_stamp);
  if constexpr (CNT) {
    // SURVEY §8(d) per-visit constants: 16 B statement record + 8 B row_ptr pair + 5 B per edge
    // (col + kind) + 8 B queue in/out (not this implementation's 64 B NodeRec / 16 B inline edges)
    const uint32_t alg_l0 = 16u + 8u + 5u * ne + 8u;
    acc_add(acc.alg, 16u * nz + 8u * nzx + 8u * hwords + (lane == 0 ? alg_l0 : 0u));
    acc_add(acc.atom, red);
    if (lane == 0) acc.dense += 8ull * B + 16ull * B * ne + alg_l0;
  }
  return cont_v;
}

// ---------------------------------------------------------------------------------- paired items
// Heavy rounds (the 4-CTA/SM instantiation): a warp takes two inline items at once, one per
// half-warp (16 lanes x 8 words = the 128-word inline limit), so every warp keeps two dependent
// load -> transfer -> union -> push chains in flight.  Same transfer and union as
// process_inline, with width-16 shuffles; IN(dst) words are loaded only where OUT is non-zero
// (no pre-read: two full pre-reads per half would not fit the register budget).
constexpr int HKW = 8;
__device__ __forceinline__ uint64_t hshfl64(uint64_t v, int src) {      // within the half-warp
  const uint32_t lo = __shfl_sync(FULL, (uint32_t)v, src, 16), hi = __shfl_sync(FULL, (uint32_t)(v >> 32), src, 16);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t half_or64(uint64_t v) {
#pragma unroll
  for (int o = 8; o; o >>= 1) v |= hshfl_xor64(v, o);
  return v;
}
__device__ __forceinline__ uint32_t half_or32(uint32_t v) {
#pragma unroll
  for (int o = 8; o; o >>= 1) v |= __shfl_xor_sync(FULL, v, o, 16);
  return v;
}
// word r of the half's block held as y[k] = word hl + 16k: r uniform in the half / per lane
__device__ __forceinline__ uint64_t huword_of(const uint64_t (&y)[HKW], uint32_t r) {
  uint64_t s = y[0];
#pragma unroll
  for (int k = 1; k < HKW; ++k) if ((r >> 4) == (uint32_t)k) s = y[k];
  return hshfl64(s, (int)(r & 15u));
}
__device__ __forceinline__ uint64_t hword_of(const uint64_t (&y)[HKW], uint32_t r) {
  uint64_t s = 0;
#pragma unroll
  for (int k = 0; k < HKW; ++k) {
    const uint64_t v = hshfl64(y[k], (int)(r & 15u));
    if ((r >> 4) == (uint32_t)k) s = v;
  }
  return s;
}

template <bool CNT>
__device__ __forceinline__ void process_inline2(const Dev& D, CtaStage& st, const NodeRec& R, const InlEdge& me,
                                                uint32_t round, uint32_t nxt, int lane, Acc& acc) {
  const int hl = lane & 15;
  const unsigned hmask = 0xffffu << (lane & 16);
  const uint32_t B = R.B, L = R.L, ne = R.n_inl, kind = R.kind;
  const uint64_t* X = D.facts + R.off;
  uint64_t y[HKW];
#pragma unroll
  for (int k = 0; k < HKW; ++k) {
    const uint32_t w = hl + 16 * k;
    y[k] = w < B ? X[w] : 0ull;
  }
  const uint32_t my_stamp = hl < (int)ne ? D.stamp[me.dst] : 1u;
  const bool is_fl = kind == GK_FLOAD || kind == GK_ALOAD, is_fs = kind == GK_FSTORE || kind == GK_ASTORE;
  const bool is_cp = kind == GK_COPY || kind == GK_SLOAD || kind == GK_RETV || kind == GK_SSTORE;
  int hr[4] = {-1, -1, -1, -1};                             // heap rows of this lane's columns
  if (is_fl || is_fs) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t c = hl + 16 * q;
      hr[q] = (c < R.n_cols) ? D.frow[R.r3 + c] : -1;
    }
  }
  // The two halves run different node kinds: every shuffle below is executed by all 32 lanes
  // (branches on warp-uniform __any_sync), each half using only its own results.
  const uint64_t row1 = huword_of(y, (is_cp || is_fl || is_fs) ? (uint32_t)R.r1 : 0u);   // rhs / w
  uint64_t row0 = 0;
  if (__any_sync(FULL, is_fs)) row0 = huword_of(y, is_fs ? (uint32_t)R.r0 : 0u);        // FSTORE base v
  int mode = 0, t = -1;
  uint64_t genv = 0;
  uint32_t fmask = 0, hwords = 0;
  if (kind == GK_PRIM || kind == GK_CONST || kind == GK_NEW) {
    mode = 1; t = R.r0;
    if (kind != GK_PRIM) genv = 1ull << (R.r3 & 63);
  } else if (is_cp) {
    mode = kind == GK_SSTORE ? 2 : 1; t = R.r0;
    genv = row1;
  } else if (is_fl) {
    mode = 1; t = R.r0;
  } else if (is_fs) {
    mode = 3;
    genv = row1;                                            // row w, OR-ed into rows (o1, f)
  }
  if (__any_sync(FULL, is_fl)) {                            // v = w.f: OR of rows (o1,f), o1 ∈ w
    uint64_t a = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t c = hl + 16 * q;
      const bool take = is_fl && hr[q] >= 0 && ((row1 >> c) & 1ull);   // NULL has no row
      const uint64_t v = hword_of(y, take ? L + (uint32_t)hr[q] : 0u);
      if (take) { a |= v; hwords += 1; }
    }
    a = half_or64(a);
    if (is_fl) genv = a;
  }
  if (__any_sync(FULL, is_fs)) {                            // v.f = w: target words of rows (o1, f)
#pragma unroll
    for (int k = 0; k < HKW; ++k) {
      uint32_t m = 0;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t c = hl + 16 * q;
        if (is_fs && hr[q] >= 0 && ((row0 >> c) & 1ull)) {
          const uint32_t w = L + (uint32_t)hr[q];
          if ((w >> 4) == (uint32_t)k) m |= 1u << (w & 15u);
        }
      }
      m = half_or32(m);
      if (is_fs && ((m >> hl) & 1u)) fmask |= 1u << k;
    }
  }
  uint32_t nzx = 0, nz = 0, red = 0;
#pragma unroll
  for (int k = 0; k < HKW; ++k) {
    const uint32_t w = hl + 16 * k;
    if (CNT) nzx += (y[k] != 0);
    if (mode == 1) { if ((int)w == t) y[k] = genv; }
    else if (mode == 2) { if ((int)w == t) y[k] |= genv; }
    else if (mode == 3) { if ((fmask >> k) & 1u) y[k] |= genv; }
  }
  unsigned gmask = 0;
#pragma unroll
  for (uint32_t i = 0; i < 4; ++i) {                        // inline edges (<= 4; per-half count)
    const bool act = i < ne;
    const uint64_t off = hshfl64(me.off, (int)i);
    const uint32_t info = __shfl_sync(FULL, me.info, (int)i, 16);
    const int kill = ((info & 3u) == GE_C2R) ? R.r0 : -1;
    uint64_t* Z = D.facts + off;
    uint64_t* zm = D.smask + (uint64_t)NMW * __shfl_sync(FULL, me.dst, (int)i, 16);
    uint64_t cur[HKW];
#pragma unroll
    for (int k = 0; k < HKW; ++k) {
      const uint32_t w = hl + 16 * k;
      cur[k] = (act && y[k] && (int)w != kill) ? Z[w] : ~0ull;
    }
    bool g = false;
#pragma unroll
    for (int k = 0; k < HKW; ++k) {
      const uint32_t w = hl + 16 * k;
      const uint64_t z = (!act || (int)w == kill) ? 0ull : y[k];
      nz += (z != 0);
      if (z & ~cur[k]) {
        red_or(Z + w, z); ++red; g = true;
        if (cur[k] == 0) nmask_note(zm, w);
      }
    }
    if (__ballot_sync(FULL, g) & hmask) gmask |= 1u << i;
  }
  flush_pushes(D, st, lane, hl < (int)ne, me.dst, me.info, (gmask >> hl) & 1u, round, nxt, nullptr, true, my_stamp);
  if constexpr (CNT) {
    const uint32_t alg_l0 = 16u + 8u + 5u * ne + 8u;       // SURVEY §8(d) constants, per item
    acc_add(acc.alg, 16u * nz + 8u * nzx + 8u * hwords + (hl == 0 ? alg_l0 : 0u));
    acc_add(acc.atom, red);
    const unsigned long long d = 8ull * B + 16ull * B * ne + alg_l0;
    const unsigned long long d2 = __shfl_sync(FULL, d, 16);
    if (lane == 0) acc.dense += d + d2;
  }
}

// ---------------------------------------------------------------------------------- one item
// The narrow part of process_item (chunk of a narrow node that is not an inline item: CALL / EXIT /
// multi-chunk nodes, blocks over the inline limit), K words per lane per pass over a block.
template <bool WIDE, bool CNT, int MW, bool CD, bool SB, int K>
__device__ __forceinline__ uint32_t narrow_item(const Dev& D, CtaStage& st, const NodeRec& R, uint32_t n, uint32_t e0,
                                             uint32_t e1, bool first, uint32_t round, uint32_t nxt, int lane,
                                             WarpScratchT<WIDE>& ws, Acc& acc, bool allow_cont, bool light,
                                             uint32_t alg_l0, uint64_t mk0, uint64_t mk1) {
  const uint32_t L = R.L, B = R.B;
  // From here on the source block is narrow (one 64-bit word per row: |Q| <= 64), in both
  // instantiations: word index = row index.
  constexpr uint32_t logW = 0u, W = 1u;
  const uint64_t* X = D.facts + R.off;             // coherent loads (no __restrict__: see process_wide)
  uint32_t cont_v = NO_CONT;                                // node to continue into (warp-uniform)

  // ---- independent loads first: this item's edge records, the first chunk of IN(src), and
  //      the rows the transfer function reads
  auto has = [&](uint32_t w) -> bool { return nmask_has(mk0, mk1, w); };
  uint64_t y[K];
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const uint32_t w = lane + 32 * k;
    y[k] = (w < B && has(w)) ? X[w] : 0ull;
  }
  const uint32_t kind = R.kind;
  int mode = 0, t = -1;                                     // 0 identity, 1 replace, 2 or-in, 3 FSTORE
  uint32_t f = 0, hwords = 0, fmask = 0;                   // fmask: FSTORE target words (bit k: word lane + 32k)
  uint64_t genv = 0;                                        // word of the generated row
  if (kind == GK_PRIM || kind == GK_CONST || kind == GK_NEW) {
    mode = 1; t = R.r0;
    if (kind != GK_PRIM) genv = 1ull << (R.r3 & 63);       // narrow: column r3 < 64
  } else if (kind == GK_COPY || kind == GK_SLOAD || kind == GK_RETV || kind == GK_SSTORE) {
    mode = kind == GK_SSTORE ? 2 : 1; t = R.r0;
    genv = X[R.r1];                                         // row rhs (all lanes: broadcast)
  } else if (kind == GK_FLOAD || kind == GK_ALOAD) {       // v = w.f: OR of rows (o1,f), o1 ∈ w
    mode = 1; t = R.r0;
    const uint64_t wrow = X[R.r1];                          // row w (all lanes: broadcast)
    int hr[2];                                              // heap rows of this lane's columns
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const uint32_t c = lane + 32 * q;
      hr[q] = (c < R.n_cols) ? D.frow[R.r3 + c] : -1;
    }
    uint64_t a = 0;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const uint32_t c = lane + 32 * q;
      if (hr[q] < 0 || !((wrow >> c) & 1ull)) continue;   // NULL has no row
      a |= X[L + hr[q]];
      hwords += 1;
    }
    genv = warp_or64(a);
  } else if (kind == GK_FSTORE || kind == GK_ASTORE) {     // v.f = w (weak)
    mode = 3; f = (uint32_t)R.r2;
    const uint64_t vrow = X[R.r0];                          // row v (all lanes: broadcast)
    genv = X[R.r1];                                         // row w, OR-ed into rows (o1, f)
    uint64_t b = vrow;
    while (b) {                                             // o1 in row v (NULL has no row)
      const int c = __ffsll((long long)b) - 1;
      b &= b - 1;
      const int hr = D.frow[R.r3 + c];
      if (hr < 0) continue;
      const uint32_t w = L + (uint32_t)hr;
      if (w < 32u * K && (w & 31u) == (uint32_t)lane) fmask |= 1u << (w >> 5);
    }
  }
  const uint64_t gsel = genv, rwsel = genv;                // identical on every lane
  (void)f;

  uint32_t nzx = 0, nz = 0, red = 0;                        // per-lane counters of this item
  unsigned long long dense_l0 = first ? 8ull * B : 0ull;
  for (uint32_t eb = e0; eb < e1; eb += 32) {               // edges in batches of 32 (a5)
    const uint32_t ne = min(32u, e1 - eb);
    const uint32_t my_info = lane < (int)ne ? D.edges[eb + lane].info : 0u;
    const uint32_t my_kind = my_info & 3u;
    const unsigned live = __ballot_sync(FULL, lane < (int)ne);
    const unsigned same = __ballot_sync(FULL, lane < (int)ne && (my_kind == GE_INTRA || my_kind == GE_C2R));
    unsigned gmask = 0;
    // -- INTRA / C2R: identical layouts; OUT computed once per chunk and reused by every edge
    if (same) {
      for (uint32_t c0 = 0; c0 < B; c0 += 32 * K) {
        if (c0 != 0 || eb != e0) {
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const uint32_t w = c0 + lane + 32 * k;
            y[k] = (w < B && has(w)) ? X[w] : 0ull;
          }
        }
#pragma unroll
        for (int k = 0; k < K; ++k) {
          const uint32_t w = c0 + lane + 32 * k;
          if (first && eb == e0) nzx += (y[k] != 0);
          if (mode == 1) { if ((int)w == t) y[k] = gsel; }
          else if (mode == 2) { if ((int)w == t) y[k] |= gsel; }
          else if (mode == 3 && c0 == 0) { if ((fmask >> k) & 1u) y[k] |= rwsel; }   // FSTORE rows (o1, f)
          else if (mode == 3) {                               // blocks of > 128 rows
            const uint32_t g = w - L;
            if (w < B && w >= L + R.n_stat && D.grow_field[R.grow_off + g] == (int)f) {
              const int c = D.grow_col[R.grow_off + g];       // o1 (never NULL)
              if ((X[R.r0] >> c) & 1ull) y[k] |= rwsel;
            }
          }
        }
        unsigned sm = same;
        while (sm) {
          const int i = __ffs(sm) - 1;
          sm &= sm - 1;
          const Edge* ep = D.edges + eb + i;
          const uint32_t info = ep->info;
          const uint64_t off = ep->off;
          const int kill = ((info & 3u) == GE_C2R) ? R.r0 : -1;     // C2R drops lhs(c)
          const uint32_t r = or_chunk(D.facts + off, y, c0, lane, kill, logW, D.smask + (uint64_t)NMW * ep->dst);
          nz += r & 0xffffu;
          red += r >> 16;
          if (r >> 16) gmask |= 1u << i;
        }
      }
      dense_l0 += 16ull * B * __popc(same);
    }
    // -- CALL / RET: layout changes (params <- args / lhs <- RET, globals, projection π)
    unsigned oth = live & ~same;
    while (oth) {
      const int i = __ffs(oth) - 1;
      oth &= oth - 1;
      const Edge* ep = D.edges + eb + i;
      const uint32_t ek = ep->info & 3u;
      const uint64_t off = ep->off;
      const uint32_t Bt = ep->B;
      const uint32_t Lt = ep->L;
      const uint32_t logWt = ep->logW;
      const int aux = ep->aux;
      const uint32_t xoff = ep->xoff;
      uint64_t* Z = D.facts + off;
      const uint32_t npar = (ek == GE_CALL) ? (uint32_t)aux : 0u;    // callee n_params
      const int lhs = (ek == GE_RET) ? aux : -1;                      // lhs(c) at the return site
      const uint32_t a0 = (ek == GE_CALL && npar > 3) ? D.arg_ptr[n] : 0u;
      // source row of target local row r (params <- args, lhs <- RET_callee), -1 = none
      auto local_src = [&](uint32_t r) -> int {
        if (ek == GE_CALL) {
          if (r >= npar) return -1;
          if (npar > 3) return D.args[a0 + r];
          return r == 0 ? R.r1 : (r == 1 ? R.r2 : R.r3);                // inline argument rows
        }
        return (int)r == lhs ? (int)(L - 1) : -1;
      };
      bool g = false;
      if (xoff == NO_XMAP) {                                // same module: word-parallel
        for (uint32_t c0 = 0; c0 < Bt; c0 += 32 * K) {
          uint64_t z[K];
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const uint32_t w = c0 + lane + 32 * k, r = w >> logW, j = w & (W - 1);
            int src = -1;
            if (w < Bt) src = (r < Lt) ? local_src(r) : (int)(L + (r - Lt));
            const uint32_t ws = ((uint32_t)src << logW) + j;
            z[k] = (src >= 0 && has(ws)) ? X[ws] : 0ull;                  // CALL/EXIT: identity
          }
          const uint32_t r = or_chunk(Z, z, c0, lane, -1, logW, D.smask + (uint64_t)NMW * ep->dst);
          nz += r & 0xffffu;
          red += r >> 16;
          if (r >> 16) g = true;
        }
        dense_l0 += 16ull * Bt;
      } else {                                              // across modules: row-parallel π
        for (uint32_t c = lane; c < R.n_cols; c += 32) ws.cmap[c] = (int16_t)D.xmap[xoff + c];
        const int32_t* rowmap = D.xmap + xoff + R.n_cols;
        const uint32_t rows_t = Bt >> logWt;
        int src[K];
#pragma unroll
        for (int k = 0; k < K; ++k) src[k] = -1;
        for (uint32_t r0 = 0; r0 < rows_t; r0 += 32 * K) {
#pragma unroll
          for (int k = 0; k < K; ++k) {                    // source row of each target row
            const uint32_t r = r0 + lane + 32 * k;
            src[k] = -1;
            if (r < rows_t) {
              if (r < Lt) src[k] = local_src(r);
              else {
                const int gs = rowmap[r - Lt];
                src[k] = gs < 0 ? -1 : (int)(L + gs);
              }
            }
          }
          __syncwarp();
          if (!WIDE || (W == 1 && logWt == 0)) {            // one word per row on both sides
            uint64_t v[K], cur[K];
#pragma unroll
            for (int k = 0; k < K; ++k) v[k] = (src[k] >= 0 && has((uint32_t)src[k])) ? X[src[k]] : 0ull;
#pragma unroll
            for (int k = 0; k < K; ++k) {
              uint64_t o = 0, b = v[k];
              while (b) {
                const int bit = __ffsll((long long)b) - 1;
                b &= b - 1;
                const int cd = ws.cmap[bit];
                if (cd >= 0) o |= 1ull << cd;
              }
              v[k] = o;
              cur[k] = o ? Z[r0 + lane + 32 * k] : ~0ull;
            }
#pragma unroll
            for (int k = 0; k < K; ++k) {
              nz += (v[k] != 0);
              if (v[k] & ~cur[k]) {
                red_or(Z + r0 + lane + 32 * k, v[k]);
                ++red;
                g = true;
                if (cur[k] == 0) nmask_note(D.smask + (uint64_t)NMW * ep->dst, r0 + lane + 32 * k);
              }
            }
          } else if constexpr (WIDE) {
#pragma unroll
            for (int k = 0; k < K; ++k) {
              if (src[k] < 0) continue;
              const uint32_t r = r0 + lane + 32 * k;
              uint64_t out[MW];
#pragma unroll
              for (int q = 0; q < MW; ++q) out[q] = 0;
              for (uint32_t j = 0; j < W; ++j) {
                uint64_t b = X[((uint64_t)src[k] << logW) + j];
                while (b) {
                  const int bit = __ffsll((long long)b) - 1;
                  b &= b - 1;
                  const int cd = ws.cmap[j * 64 + bit];
                  if (cd < 0) continue;
#pragma unroll
                  for (int q = 0; q < MW; ++q)
                    if (q == (cd >> 6)) out[q] |= 1ull << (cd & 63);
                }
              }
              emit_row_words(Z, Bt, logWt, r, out, nz, red, g, D.smask + (uint64_t)NMW * ep->dst, D.delta + off);   // occupancy, Δ
            }
          }
        }
        __syncwarp();
        dense_l0 += 16ull * Bt;
      }
      if (g) gmask |= 1u << i;
    }
    const unsigned gall = __reduce_or_sync(FULL, gmask);
    const uint32_t my_dst = lane < (int)ne ? D.edges[eb + lane].dst : 0u;
    flush_pushes<SB>(D, st, lane, lane < (int)ne, my_dst, my_info, (gall >> lane) & 1u, round, nxt,
                 (CD && allow_cont && light) ? &cont_v : nullptr, true);
  }
  if constexpr (CNT) {
    acc_add(acc.alg, 16u * nz + 8u * nzx + 8u * hwords + (lane == 0 ? alg_l0 : 0u));
    acc_add(acc.atom, red);
    if (lane == 0) acc.dense += dense_l0 + alg_l0;
  }
  return cont_v;
}


template <bool WIDE, bool CNT, int MW, bool CD, bool SB = false>
__device__ uint32_t process_item(const Dev& D, CtaStage& st, uint32_t n, uint32_t ci, uint32_t round,
                                 uint32_t nxt, int lane, WarpScratchT<WIDE>& ws, Acc& acc, bool allow_cont,
                                 bool light = false) {
  const uint64_t mk0 = GD_NMASK ? D.smask[(uint64_t)NMW * n] : ~0ull;       // (issued with the NodeRec load)
  const uint64_t mk1 = GD_NMASK ? D.smask[(uint64_t)NMW * n + 1] : ~0ull;
  const NodeRec R = D.nodes[n];
  InlEdge me{0u, 0u, 0ull};                                 // inline chunk-0 edge of this lane (same hop)
  if (GD_INL && !WIDE && lane < 4) me = D.inl[4 * n + lane];
  const uint32_t deg = R.e1 - R.e0, ebs = chunk_edges(deg, R.cls, R.logW);
  const uint32_t e0 = R.e0 + ci * ebs, e1 = min(R.e1, e0 + ebs);
  const bool first = ci == 0;
  const uint32_t L = R.L, B = R.B;
  // SURVEY §8(d) constants: statement record + row_ptr once per node visit (chunk 0), 5 B per
  // edge, 8 B queue entry in/out per item
  uint32_t alg_l0 = (first ? 16u + 8u : 0u) + 5u * (e1 - e0) + 8u;
  if (e0 >= e1) {                                           // no successor: nothing to propagate
    if (CNT && lane == 0) { acc.alg += alg_l0; acc.dense += alg_l0; }
    return NO_CONT;
  }
  if constexpr (WIDE) {
    if (R.logW >= 1) {                                      // wide block: row-sparse path
      uint32_t cont_v = NO_CONT;                            // node to continue into (warp-uniform)
      process_wide<CNT, MW, SB>(D, st, R, n, e0, e1, first, round, nxt, lane, ws, acc, alg_l0,
                   (GD_CONT_WIDE && allow_cont) ? &cont_v : nullptr, CD && light);
      return cont_v;
    }
  }
  if (GD_INL && !WIDE && first && R.n_inl && (GD_INL4 || R.B <= 96u)) {   // (wide batches: measured slower)
    if (GD_INL2 && R.B <= 64u)                             // every row in words 0..63: 2 per lane
      return process_inline<CNT, CD, SB, 2>(D, st, R, me, round, nxt, lane, acc, allow_cont && light, mk0, mk1);
    if (GD_INL3 && R.B <= 96u)                             // every row in words 0..95: 3 per lane
      return process_inline<CNT, CD, SB, 3>(D, st, R, me, round, nxt, lane, acc, allow_cont && light, mk0, mk1);
    return process_inline<CNT, CD, SB>(D, st, R, me, round, nxt, lane, acc, allow_cont && light, mk0, mk1);
  }
  if (!WIDE && GD_ITEM3 && B <= 96u)
    return narrow_item<WIDE, CNT, MW, CD, SB, 3>(D, st, R, n, e0, e1, first, round, nxt, lane, ws, acc, allow_cont,
                                                 light, alg_l0, mk0, mk1);
  return narrow_item<WIDE, CNT, MW, CD, SB, KW>(D, st, R, n, e0, e1, first, round, nxt, lane, ws, acc, allow_cont,
                                                light, alg_l0, mk0, mk1);
}

// ---------------------------------------------------------------------------------- rounds
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
      while (*vgen == gen) {
        if constexpr (GD_BAR_NS > 0) __nanosleep(GD_BAR_NS);
      }
    }
    __threadfence();                       // acquire: later loads see other SMs' writes
  }
  __syncthreads();
}

__device__ __forceinline__ void flush_acc(const Dev& D, const Acc& acc) {
  if ((threadIdx.x & 31) == 0 && (acc.alg | acc.atom | acc.dense | acc.cont)) {
    atomicAdd(&D.stats->visits, acc.cont);
    atomicAdd(&D.stats->alg_bytes, acc.alg);
    atomicAdd(&D.stats->atomics, acc.atom);
    atomicAdd(&D.stats->dense_bytes, acc.dense);
  }
}

// Process every item of round `round` with warps gw, gw+nw, ...; returns total items (0 when
// the worklist is empty: the fixed point of Alg. 1 l.10 is reached).
template <bool WIDE, bool CNT, int MW, bool CD, bool PAIR = false>
__device__ __forceinline__ uint32_t run_round(const Dev& D, CtaStage& st, uint32_t round, uint32_t gw,
                                              uint32_t nw, int lane, WarpScratchT<WIDE>& ws, Acc& acc) {
  const uint32_t cur = round % 3, nxt = (round + 1) % 3, clr = (round + 2) % 3;
  uint32_t cnt[NCLS];
  uint32_t total = 0;
  if (D.bar[BAR_DONE]) return 0;          // an earlier round found the worklist empty
#pragma unroll
  for (int c = 0; c < NCLS; ++c) { cnt[c] = D.counts[cur * CNT_STRIDE + c]; total += cnt[c]; }
  if (total == 0) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      D.bar[BAR_DONE] = 1;
      if (round <= D.trace_cap) {
        unsigned long long ns;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ns));
        D.trace[2 * (round - 1)] = ns;
        D.trace[2 * (round - 1) + 1] = 0;
      }
    }
    return 0;
  }
  if (D.max_rounds && round > D.max_rounds) return total;
  if ((D.sw_lo && total < D.sw_lo) || (D.sw_hi && total >= D.sw_hi)) {   // hybrid: hand over
    if (blockIdx.x == 0 && threadIdx.x == 0) D.bar[3] = round;
    return ROUND_SWITCH;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const uint32_t nodes = D.counts[cur * CNT_STRIDE + CNT_NODES];
#pragma unroll
    for (int c = 0; c < CNT_STRIDE; ++c) D.counts[clr * CNT_STRIDE + c] = 0;
    // atomics: in loop_mode 1 other CTAs of this launch may already add continuation visits
    atomicAdd(&D.stats->rounds, 1ull);
    atomicAdd(&D.stats->visits, (unsigned long long)nodes);
    atomicAdd(&D.stats->hist[nodes <= 32 ? 0 : (nodes <= 64 ? 1 : 2)], 1ull);
    if (round <= D.trace_cap) {
      unsigned long long ns;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ns));
      D.trace[2 * (round - 1)] = ns;
      D.trace[2 * (round - 1) + 1] = ((unsigned long long)total << 32) | nodes;
    }
  }
  const uint32_t* Q = D.queue + (size_t)cur * D.n_chunks;
  const uint32_t b1 = cnt[0], b2 = b1 + cnt[1], b3 = b2 + cnt[2], b4 = b3 + cnt[3];   // class boundaries
  auto entry_of = [&](uint32_t item) -> uint32_t {          // item -> class segment -> entry
    const uint32_t c = (item >= b1) + (item >= b2) + (item >= b3) + (item >= b4);
    const uint32_t base = c == 0 ? 0u : (c == 1 ? b1 : (c == 2 ? b2 : (c == 3 ? b3 : b4)));
    return Q[D.seg[c] + (item - base)];
  };
  // Continuation into narrow destinations (GD_CONT_DENSE) only while the round leaves warps
  // idle (total items below GD_CONT_LOAD/4 x warps); wide destinations always continue.
  // Narrow continuation (CD) is compiled into the 3-CTA/SM narrow instantiation only: small
  // and median apps spend most rounds light (small 2.30 -> 1.92 ms, 332 -> 80 rounds; median
  // 6.59 -> 6.31 ms), while the corpus shard (+7 %) and wide batches (+1 %) lost with it.
  const bool cont_ok = (uint64_t)total * 4u < (uint64_t)nw * GD_CONT_LOAD;
  // MER (Fig. 7): process the head list — whole waves of nw items — and
  // merge the tail into the next worklist (the round stamp removes repetitions).
  const uint32_t head = ((D.flags & F_MER) && total > nw) ? (total / nw) * nw : total;
  if constexpr (PAIR) {
    // heavy rounds (4-CTA/SM instantiation, no continuation, no MER): two items per warp; a pair
    // of inline items runs on the two half-warps, any other pair item by item on the full warp
    if (!(D.flags & F_MER)) {
      for (uint32_t item = gw; item < total; item += 2 * nw) {
        const uint32_t item2 = item + nw;
        const bool has2 = item2 < total;
        const uint32_t ea = entry_of(item), eb = has2 ? entry_of(item2) : ea;
        const uint32_t my_e = (lane >= 16 && has2) ? eb : ea;
        const uint32_t my_n = my_e >> 5;
        const NodeRec R = D.nodes[my_n];
        InlEdge me{0u, 0u, 0ull};
        if ((lane & 15) < 4) me = D.inl[4 * my_n + (lane & 15)];
        const bool elig = (my_e & 31u) == 0 && R.n_inl != 0;
        if (has2 && __all_sync(FULL, elig)) {
          process_inline2<CNT>(D, st, R, me, round, nxt, lane, acc);
        } else {
          process_item<WIDE, CNT, MW, CD>(D, st, ea >> 5, ea & 31u, round, nxt, lane, ws, acc, false);
          if (has2) process_item<WIDE, CNT, MW, CD>(D, st, eb >> 5, eb & 31u, round, nxt, lane, ws, acc, false);
        }
      }
      return total;
    }
  }
  // Wide batches (GD_DYN): item costs differ by orders of magnitude (a wide node is visited
  // whole, over every out-edge), so after its first item a warp takes the next unclaimed one from
  // a per-round counter (counts slot 6 of this rotation, cleared with the others) instead of
  // striding by the warp count; a warp that drew heavy items no longer holds the round open.
  // Dynamic hand-out (GD_DYN: wide batches; GD_DYN_NARROW: narrow ones): item costs differ by
  // orders of magnitude (a wide node is visited whole, over every out-edge; a CALL or EXIT chunk
  // remaps a whole block), so after its first item a warp takes the next unclaimed one from a
  // per-round counter (counts slot 6 of this rotation, cleared with the others) instead of
  // striding by the warp count, and a warp that drew heavy items no longer holds the round open.
  // The claim for the item after next is issued one item ahead (lane 0 holds it until the
  // broadcast), so its latency hides behind the current item.  A warp's claims increase, so a
  // claimed index < total is always processed by its claimer.
  // Narrow rounds claim GD_DYN_GRAIN consecutive items per atomic (one counter for ~100M items
  // per build is a hotspot at grain 1).
  const bool dyn = GD_DYN && (WIDE || GD_DYN_NARROW) && total > nw;
  constexpr uint32_t G = WIDE ? 1u : (uint32_t)GD_DYN_GRAIN;
  uint32_t* const ctr = D.counts + cur * CNT_STRIDE + 6;
  uint32_t item = gw, nitem = gw + nw, nend = 0;                     // nend: end of nitem's claim
  if (dyn) {
    uint32_t v = 0;
    if (lane == 0) v = nw + G * atomicAdd(ctr, 1u);
    nitem = __shfl_sync(FULL, v, 0);
    nend = nitem + G;
  }
  auto advance = [&](uint32_t pend) {                                // item <- nitem <- the one after
    item = nitem;
    if (!dyn) nitem += nw;
    else if (nitem + 1 < nend) ++nitem;
    else { nitem = __shfl_sync(FULL, pend, 0); nend = nitem + G; }
  };
  uint32_t entry = item < total ? entry_of(item) : 0u;
  while (item < total) {
    uint32_t pend = 0;                          // lane 0: the next claim, issued one item ahead
    if (dyn && nitem + 1 >= nend && lane == 0) pend = nw + G * atomicAdd(ctr, 1u);
    if (item >= head) {                                                // tail: defer to round+1
      const uint32_t n = entry >> 5;
      uint32_t info = 0;
      if (lane == 0) {
        const NodeRec R = D.nodes[n];
        info = ((uint32_t)R.cls << 2) | ((n_chunks_of(R.e1 - R.e0, R.cls, R.logW) - 1) << 5);
      }
      flush_pushes(D, st, lane, lane == 0, n, info, true, round, nxt);
      advance(pend);
      entry = item < total ? entry_of(item) : 0u;
      continue;
    }
    const uint32_t nentry = nitem < total ? entry_of(nitem) : 0u;    // prefetch the next item
    if constexpr (GD_PF) {
      // two-stage software pipeline: the records of item i+2 into L1, and — from item i+1's
      // records, prefetched one iteration ago — the lines of its IN(src) and of the first two
      // IN(dst) blocks into L2, all before item i's own chain starts
      const uint32_t n2item = nitem + nw;
      if (n2item < total && lane < 2) {
        const uint32_t nn2 = entry_of(n2item) >> 5;
        asm volatile("prefetch.global.L1 [%0];" :: "l"(lane == 0 ? (const char*)(D.nodes + nn2) : (const char*)(D.inl + 4 * nn2)));
      }
      if (nitem < total && lane < 24 && (nentry & 31u) == 0) {
        const uint32_t nn = nentry >> 5;
        const uint32_t Bn = D.nodes[nn].B, line = lane & 7u;
        if (D.nodes[nn].logW == 0 && line * 16u < Bn) {
          const uint32_t which = lane >> 3;                  // 0: IN(src), 1-2: IN(dst) of inline edges
          const uint64_t o = which == 0 ? D.nodes[nn].off
                                        : (which <= D.nodes[nn].n_inl ? D.inl[4 * nn + which - 1].off : ~0ull);
          if (o != ~0ull) asm volatile("prefetch.global.L2 [%0];" :: "l"((const char*)(D.facts + o + line * 16u)));
        }
      }
    } else if (nitem < total && lane < 2) {                            // NodeRec, inline edges into L1
      const uint32_t nn = nentry >> 5;
      asm volatile("prefetch.global.L1 [%0];" :: "l"(lane == 0 ? (const char*)(D.nodes + nn) : (const char*)(D.inl + 4 * nn)));
    }
    if constexpr (GD_CONT_DEPTH == 0 || (!WIDE && !CD)) {
      process_item<WIDE, CNT, MW, CD>(D, st, entry >> 5, entry & 31u, round, nxt, lane, ws, acc, false);
    } else {
      uint32_t n = entry >> 5, ci = entry & 31u;
      for (int depth = 0;; ++depth) {
        const uint32_t c = process_item<WIDE, CNT, MW, CD>(D, st, n, ci, round, nxt, lane, ws, acc,
                                              depth < (WIDE ? GD_CONT_DEPTH : GD_CONT_DEPTH_NARROW), cont_ok);
        if (c == NO_CONT) break;
        __syncwarp();                      // this warp's ORs into IN(c) are visible to all lanes
        if constexpr (WIDE) __threadfence();   // + its Δ(c) bits (the visit consumes them): L2 order
        else __threadfence_block();
        n = c;
        ci = 0;
        if (lane == 0) acc.cont += 1;
      }
    }
    advance(pend);
    entry = nentry;
  }
  return total;
}

template <bool WIDE, bool CNT, int MW, int MINB>
__global__ void __launch_bounds__(THREADS, MINB) k_fixpoint(Dev D) {
  __shared__ WarpScratchT<WIDE> ws_all[WARPS];
  __shared__ Acc acc_all[WARPS];
  __shared__ CtaStage st;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * WARPS + wib, nw = gridDim.x * WARPS;
  Acc& acc = acc_all[wib];
  if (lane == 0) acc = Acc{0, 0, 0, 0};
  stage_init(st);
  uint32_t round0 = D.round0;
  if (D.hyb) {                 // hybrid sequence: resume where the previous launch handed over
    round0 = *(volatile uint32_t*)(D.bar + 3);
    if (round0 == 0) return;   // (uniform: bar[3] changes only when this launch ends, see below)
  }
  __syncthreads();
  for (uint32_t round = round0;; ++round) {
    const uint32_t total = run_round<WIDE, CNT, MW, GD_CONT_DENSE && !WIDE && (MINB == GD_MINB || GD_CD_HI),
                                     GD_PAIR && !WIDE && MINB == GD_MINB_HI>(D, st, round, gw, nw, lane, ws_all[wib], acc);
    if (total == ROUND_SWITCH) break;                 // bar[3] = this round (run_round)
    if (total == 0) {                                 // fixed point: later launches return at once
      if (D.hyb && blockIdx.x == 0 && threadIdx.x == 0) D.bar[3] = 0;
      break;
    }
    if (D.max_rounds && round > D.max_rounds) {
      if (blockIdx.x == 0 && threadIdx.x == 0) {
        D.stats->limit_hit = 1;
        if (D.hyb) D.bar[3] = 0;
      }
      break;
    }
    stage_publish(D, st, (round + 1) % 3);
    grid_sync(D.bar, gridDim.x);
  }
  flush_acc(D, acc);
}

template <bool WIDE, bool CNT, int MW>
__global__ void __launch_bounds__(THREADS, GD_MINB) k_round(Dev D, uint32_t round) {
  __shared__ WarpScratchT<WIDE> ws_all[WARPS];
  __shared__ Acc acc_all[WARPS];
  __shared__ CtaStage st;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * WARPS + wib, nw = gridDim.x * WARPS;
  Acc& acc = acc_all[wib];
  if (lane == 0) acc = Acc{0, 0, 0, 0};
  stage_init(st);
  __syncthreads();
  const uint32_t total = run_round<WIDE, CNT, MW, GD_CONT_DENSE && !WIDE>(D, st, round, gw, nw, lane, ws_all[wib],
                                                                         acc);
  if (total == ROUND_SWITCH) { flush_acc(D, acc); return; }
  if (total && D.max_rounds && round > D.max_rounds && blockIdx.x == 0 && threadIdx.x == 0)
    D.stats->limit_hit = 1;
  if (total) stage_publish(D, st, (round + 1) % 3);
  flush_acc(D, acc);
}

// ---------------------------------------------------------------------------------- SBDA
// The paper's two-level decomposition (§III-A2, Fig. 3; Alg. 2 l.6 "mid <-
// blockIdx.x"): one CTA per method, its threads running the method's worklist.  On B200 a
// pass claims every method with queued nodes (the global worklist, one entry per node) for one
// CTA; the CTA solves that method to local quiescence in shared-memory worklists with
// __syncthreads between local rounds (no grid barrier), INTRA/C2R successors staying local;
// CALL/RET successors — the interprocedural hops a method summary would stand for — go to the
// global worklist of the next pass.  Passes end at an empty worklist.  Same least fixed point
// (any fair chaotic iteration, DESIGN.md §3 C4 / reading R8); visits = local items processed.
template <bool WIDE, bool CNT, int MW>
__global__ void __launch_bounds__(THREADS, GD_MINB) k_sbda(Dev D) {
  __shared__ WarpScratchT<WIDE> ws_all[WARPS];
  __shared__ Acc acc_all[WARPS];
  __shared__ CtaStage st;
  __shared__ uint32_t lq[2 * LQCAP];
  __shared__ uint32_t s_m, s_go;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  Acc& acc = acc_all[wib];
  if (lane == 0) acc = Acc{0, 0, 0, 0};
  stage_init(st);
  if (threadIdx.x == 0) st.lq = lq;
  __syncthreads();
  uint32_t counter = 0;
  for (uint32_t pass = D.round0;; ++pass) {
    const uint32_t cur = pass % 3, nxt = (pass + 1) % 3, clr = (pass + 2) % 3;
    if (D.bar[BAR_DONE]) break;
    uint32_t cnt[NCLS], total = 0;
#pragma unroll
    for (int c = 0; c < NCLS; ++c) { cnt[c] = D.counts[cur * CNT_STRIDE + c]; total += cnt[c]; }
    if (total == 0) {
      if (blockIdx.x == 0 && threadIdx.x == 0) D.bar[BAR_DONE] = 1;
      break;
    }
    if (D.max_rounds && pass > D.max_rounds) {
      if (blockIdx.x == 0 && threadIdx.x == 0) D.stats->limit_hit = 1;
      break;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
#pragma unroll
      for (int c = 0; c < CNT_STRIDE; ++c) D.counts[clr * CNT_STRIDE + c] = 0;
      D.bar[4 + nxt] = 0;                                   // claim cursor of the next pass
      atomicAdd(&D.stats->rounds, 1ull);
      const uint32_t nodes = D.counts[cur * CNT_STRIDE + CNT_NODES];
      atomicAdd(&D.stats->hist[nodes <= 32 ? 0 : (nodes <= 64 ? 1 : 2)], 1ull);
    }
    const uint32_t* Q = D.queue + (size_t)cur * D.n_chunks;
    const uint32_t b1 = cnt[0], b2 = b1 + cnt[1], b3 = b2 + cnt[2], b4 = b3 + cnt[3];
    for (;;) {
      if (threadIdx.x == 0) {                               // claim the next queued node's method
        const uint32_t i = atomicAdd(&D.bar[4 + cur], 1u);
        s_go = i < total;
        s_m = 0xffffffffu;
        if (i < total) {
          const uint32_t c = (i >= b1) + (i >= b2) + (i >= b3) + (i >= b4);
          const uint32_t base = c == 0 ? 0u : (c == 1 ? b1 : (c == 2 ? b2 : (c == 3 ? b3 : b4)));
          const uint32_t n = Q[D.seg[c] + (i - base)] >> 5;
          const uint32_t m = D.node_method[n];
          if (atomicExch(&D.claim[m], pass) != pass) s_m = m;
        }
        st.lsel = 0;
        st.lcnt[0] = st.lcnt[1] = 0;
        st.lid = ((unsigned long long)pass << 32) | ++counter;
      }
      __syncthreads();
      if (!s_go) break;
      const uint32_t m = s_m;
      if (m != 0xffffffffu) {
        // local worklist 0: the method's nodes queued for this pass (all their chunks)
        const uint32_t p0 = D.meth_node_ptr[m], p1 = D.meth_node_ptr[m + 1];
        for (uint32_t t = p0 + threadIdx.x; t < p1; t += THREADS) {
          const uint32_t n = D.meth_nodes[t];
          if (D.stamp[n] != pass) continue;
          const NodeRec R = D.nodes[n];
          const uint32_t nch = n_chunks_of(R.e1 - R.e0, R.cls, R.logW);
          const uint32_t base = atomicAdd(&st.lcnt[0], nch);
          if (base + nch <= LQCAP) {
            for (uint32_t q = 0; q < nch; ++q) lq[base + q] = (n << 5) | q;
          } else {                                          // local queue full: the next pass
            for (uint32_t q = base; q < LQCAP; ++q) lq[q] = LQ_SKIP;
            if (atomicMax(&D.stamp[n], pass + 1) < pass + 1) {
              const uint32_t cls = (D.flags & F_GRP) ? R.cls : 0u;
              const uint32_t g = atomicAdd(&D.counts[nxt * CNT_STRIDE + cls], nch);
              for (uint32_t q = 0; q < nch; ++q) D.queue[(size_t)nxt * D.n_chunks + D.seg[cls] + g + q] = (n << 5) | q;
              atomicAdd(&D.counts[nxt * CNT_STRIDE + CNT_NODES], 1u);
            }
          }
        }
        __syncthreads();
        for (;;) {                                          // local rounds (Alg. 2 l.7-18 in one block)
          const uint32_t sel = st.lsel;
          const uint32_t ni = min(st.lcnt[sel], LQCAP);
          if (ni == 0) break;
          for (uint32_t it = wib; it < ni; it += WARPS) {
            const uint32_t e = lq[sel * LQCAP + it];
            if (e == LQ_SKIP) continue;
            process_item<WIDE, CNT, MW, false, true>(D, st, e >> 5, e & 31u, pass, nxt, lane, ws_all[wib], acc, false);
            if (lane == 0) acc.cont += 1;                   // a visit (stats->visits)
          }
          __syncthreads();
          if (threadIdx.x == 0) {
            st.lcnt[sel] = 0;
            st.lsel = sel ^ 1u;
            st.lid = ((unsigned long long)pass << 32) | ++counter;
          }
          __syncthreads();
        }
      }
      __syncthreads();
    }
    stage_publish(D, st, nxt);
    grid_sync(D.bar, gridDim.x);
  }
  flush_acc(D, acc);
}

// method -> nodes CSR for the SBDA schedule (counts, one-block scan, fill)
__global__ void k_meth_count(Dev D, uint32_t* cnt) {
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < D.n_nodes; n += gridDim.x * blockDim.x)
    atomicAdd(&cnt[D.node_method[n] + 1], 1u);
}
__global__ void k_meth_scan(uint32_t* ptr, uint32_t M) {   // inclusive scan of ptr[1..M], one block
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint32_t b = 0; b < M; b += blockDim.x) {
    const uint32_t i = b + threadIdx.x + 1;
    uint32_t v = i <= M ? ptr[i] : 0u;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) { const uint32_t t = __shfl_up_sync(FULL, v, o); if (lane >= o) v += t; }
    __shared__ uint32_t ws[32];
    if (lane == 31) ws[w] = v;
    __syncthreads();
    if (w == 0) {
      uint32_t x = lane < (int)(blockDim.x >> 5) ? ws[lane] : 0u;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) { const uint32_t t = __shfl_up_sync(FULL, x, o); if (lane >= o) x += t; }
      ws[lane] = x;
    }
    __syncthreads();
    v += (w ? ws[w - 1] : 0u) + carry;
    if (i <= M) ptr[i] = v;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = v;
    __syncthreads();
  }
}
__global__ void k_meth_fill(Dev D, const uint32_t* ptr, uint32_t* cursor, uint32_t* nodes) {
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < D.n_nodes; n += gridDim.x * blockDim.x) {
    const uint32_t m = D.node_method[n];
    nodes[ptr[m] + atomicAdd(&cursor[m], 1u)] = n;
  }
}

// (a1) Rebase the staged app-local node tables by their app's bases (NodeRec::app).
__global__ void k_rebase(Dev D, NodeRec* nodes, uint32_t* nodemeth, uint32_t* rowptr, uint32_t* argptr,
                         const AppBase* __restrict__ bases) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < D.n_nodes; n += stride) {
    NodeRec R = nodes[n];
    const AppBase b = bases[R.app];
    R.off += b.fact; R.e0 += b.edge; R.e1 += b.edge;
    R.col_off += b.col; R.grow_off += b.grow;
    if (R.kind >= GK_FLOAD && R.kind <= GK_ASTORE && R.r3 >= 0) R.r3 += (int32_t)b.frow;
    nodes[n] = R;
    nodemeth[n] += b.meth;
    rowptr[n + 1] += b.edge;
    argptr[n + 1] += b.args;
  }
}

// (a1) Edge records (destination layout copied in) and the inline chunk-0 records, one thread
// per source node: col is app-local, so the destination id is app_node_base[app] + col[e].
// CALL aux = the callee's n_params (its ENTRY NodeRec holds it in r1); RET aux = lhs(c) of the
// return site (its r0).  Chunk 0 goes inline when it holds only INTRA/C2R edges of a narrow
// block of <= INL_MAX_B words.
__global__ void k_edges(Dev D, Edge* edges, InlEdge* inl, NodeRec* nodes, const uint32_t* __restrict__ ecol,
                        const uint8_t* __restrict__ ekind, const uint32_t* __restrict__ exoff) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < D.n_nodes; n += stride) {
    const NodeRec R = nodes[n];
    const uint32_t base = D.app_node_base[R.app];
    const uint32_t deg = R.e1 - R.e0, n0 = min(deg, chunk_edges(deg, R.cls, R.logW));
    bool inl_ok = deg > 0 && n0 <= 4 && R.logW == 0 && R.B <= INL_MAX_B;
    InlEdge rec[4];
    for (uint32_t e = R.e0; e < R.e1; ++e) {
      const uint32_t s = base + ecol[e], ek = ekind[e];
      const NodeRec& RS = nodes[s];
      const uint32_t cls = RS.cls, logW = RS.logW;
      const uint32_t nch = n_chunks_of(RS.e1 - RS.e0, cls, logW);
      Edge E2;
      E2.dst = s;
      E2.info = ek | (cls << 2) | ((nch - 1) << 5) | (logW >= 1 ? INFO_WIDE : 0u);
      E2.off = RS.off; E2.B = RS.B; E2.L = (uint16_t)RS.L; E2.logW = (uint8_t)logW; E2.pad = 0;
      E2.aux = ek == GE_CALL ? RS.r1 : (ek == GE_RET ? RS.r0 : -1);
      E2.xoff = exoff[e];
      edges[e] = E2;
      const uint32_t j = e - R.e0;
      if (j < 4) rec[j] = InlEdge{E2.dst, E2.info, E2.off};
      if (j < n0) inl_ok = inl_ok && (ek == GE_INTRA || ek == GE_C2R);
    }
    for (uint32_t j = 0; j < 4; ++j) inl[4 * n + j] = (inl_ok && j < n0) ? rec[j] : InlEdge{0u, 0u, 0ull};
    nodes[n].n_inl = inl_ok ? (uint8_t)n0 : (uint8_t)0;   // (other threads read other fields only)
  }
}

// (a2) seed round 1 with the component entries (Alg. 1 l.9)
__global__ void k_seed(Dev D) {
  // The first round of this build is D.round0 (1, or after the rounds of earlier builds of an
  // incremental handle): entries (fresh builds) and staged seed nodes (gdroid_stage_seeds) are
  // queued for it, stamped round0, in queue slot round0 % 3.
  __shared__ CtaStage st;
  const int lane = threadIdx.x & 31;
  const uint32_t r0 = D.round0;
  stage_init(st);
  __syncthreads();
  const uint32_t ne = D.push_entries ? D.n_entries : 0u, nt = ne + D.n_seed_nodes;
  for (uint32_t i0 = 0; i0 < nt; i0 += 32) {
    const uint32_t i = i0 + lane;
    const bool act = i < nt;
    const uint32_t e = act ? (i < ne ? D.entries[i] : D.seed_nodes[i - ne]) : 0u;
    uint32_t info = 0;
    if (act) {
      const NodeRec R = D.nodes[e];
      info = ((uint32_t)R.cls << 2) | ((n_chunks_of(R.e1 - R.e0, R.cls, R.logW) - 1) << 5);
    }
    flush_pushes(D, st, lane, act, e, info, true, r0 - 1, r0 % 3);
  }
  stage_publish(D, st, r0 % 3);
  if (threadIdx.x == 0) D.bar[3] = r0;    // hybrid sequences start here
}

// Staged seed facts (gdroid_stage_seeds): OR pair (slot gid, instance gid) into IN(node) —
// and into Δ(node) and the row-occupancy bitmap for wide blocks — before the build's first
// round.  One thread per pair: slot -> row (method local, else binary search of the module's
// ascending global-row gids), instance -> column (binary search of the sorted pool).  A pair
// outside the node's pools P_m x Q_m sets stats->seed_err (GDROID_E_POOL).
__global__ void k_apply_seeds(Dev D) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= D.n_seed_pairs) return;
  const uint32_t node = D.seed_pairs[3 * i], slot = D.seed_pairs[3 * i + 1], inst = D.seed_pairs[3 * i + 2];
  const NodeRec R = D.nodes[node];
  const uint32_t L = R.L, rows = R.B >> R.logW;
  int64_t row = -1;
  if (slot - R.local_base < L) row = slot - R.local_base;
  else {
    uint32_t lo = 0, hi = rows - L;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (D.grow_gid[R.grow_off + mid] < slot) lo = mid + 1; else hi = mid;
    }
    if (lo < rows - L && D.grow_gid[R.grow_off + lo] == slot) row = L + lo;
  }
  uint32_t lo = 0, hi = R.n_cols;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (D.col_gid[R.col_off + mid] < inst) lo = mid + 1; else hi = mid;
  }
  if (row < 0 || lo >= R.n_cols || D.col_gid[R.col_off + lo] != inst) {
    atomicExch(&D.stats->seed_err, 1ull + i);
    return;
  }
  const uint64_t w = ((uint64_t)row << R.logW) + (lo >> 6), bit = 1ull << (lo & 63);
  atomicOr((unsigned long long*)(D.facts + R.off + w), bit);
  if (R.logW >= 1) {
    atomicOr((unsigned long long*)(D.delta + R.off + w), bit);
    atomicOr((unsigned long long*)(D.facts + R.off + occ_offset(R.B) + (row >> 6)), 1ull << (row & 63));
  } else if (GD_NMASK && w < 64u * NMW) {
    atomicOr((unsigned long long*)(D.smask + (uint64_t)NMW * node + (w >> 6)), 1ull << (w & 63));
  }
}

// Narrow word-occupancy masks from the facts themselves (after gdroid_import_facts).
__global__ void k_nmask_rebuild(Dev D) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < D.n_nodes; n += nw) {
    const NodeRec R = D.nodes[n];
    if (R.logW != 0) continue;
#pragma unroll
    for (uint32_t q = 0; q < NMW; ++q) {
      const uint32_t w0 = q * 64 + lane, w1 = w0 + 32;
      const bool a = w0 < R.B && D.facts[R.off + w0] != 0, b = w1 < R.B && D.facts[R.off + w1] != 0;
      const uint64_t m = (uint64_t)__ballot_sync(FULL, a) | ((uint64_t)__ballot_sync(FULL, b) << 32);
      if (lane == 0) D.smask[(uint64_t)NMW * n + q] = m;
    }
  }
}

// (a7) per-node digests d(n) = Σ mix64(mix64(n) ^ (slot<<32 | inst)) (C8).  A warp's nodes are
// nw apart, so consecutive ones almost always belong to the same app: the app sum is carried in
// a register and added once per app change (not one same-address atomic per node).
// Digest of one node's block held as y[k] = word lane + 32k (k < DKW), plus any words beyond.
constexpr int DKW = 4;
__device__ __forceinline__ unsigned long long digest_words(const Dev& D, const NodeRec& R, uint64_t hn,
                                                           const uint64_t (&y)[DKW], int lane, uint32_t& pc) {
  const uint32_t logW = R.logW, L = R.L, B = R.B, jm = (1u << logW) - 1;
  unsigned long long s = 0;
  auto one = [&](uint32_t w, uint64_t x) {
    const uint32_t r = w >> logW, j = w & jm;
    const uint64_t slot = r < L ? (uint64_t)(R.local_base + r) : (uint64_t)D.grow_gid[R.grow_off + r - L];
    const uint64_t hs = hn ^ (slot << 32);
    const uint32_t* cg = D.col_gid + R.col_off + j * 64;
    if constexpr (GD_DIG_U2) {
      // two bits per iteration: both column loads and both hashes in flight together
      while (x) {
        const int b0 = __ffsll((long long)x) - 1;
        x &= x - 1;
        if (x) {
          const int b1 = __ffsll((long long)x) - 1;
          x &= x - 1;
          const uint64_t o0 = cg[b0], o1 = cg[b1];
          s += mix64(hs ^ o0) + mix64(hs ^ o1);
        } else {
          s += mix64(hs ^ (uint64_t)cg[b0]);
        }
      }
    } else {
      while (x) {
        const int b = __ffsll((long long)x) - 1;
        x &= x - 1;
        const uint64_t o = cg[b];
        s += mix64(hs ^ o);
      }
    }
  };
#pragma unroll
  for (int k = 0; k < DKW; ++k)
    if (y[k]) one(lane + 32 * k, y[k]);
  const uint64_t* X = D.facts + R.off;
  if (logW >= 1) {                                         // wide block: occupied rows only
    const uint32_t rows = B >> logW, nocc = occ_words(rows), W = 1u << logW;
    const uint64_t* X = D.facts + R.off;
    const uint64_t* OCC = X + occ_offset(B);
    for (uint32_t i = 0; i < nocc; ++i) {
      const uint64_t ow = OCC[i];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint32_t j = (uint32_t)lane + 32u * h;
        if (!((ow >> j) & 1ull)) continue;
        const uint32_t r = i * 64 + j;
        for (uint32_t q = 0; q < W; ++q) {
          const uint32_t w = (r << logW) + q;
          const uint64_t x = X[w];
          pc += __popcll(x);
          if (x) one(w, x);
        }
      }
    }
    return s;
  }
#pragma unroll
  for (int k = 0; k < DKW; ++k) pc += __popcll(y[k]);
  for (uint32_t w = lane + 32 * DKW; w < B; w += 32) {     // blocks beyond 128 words (narrow)
    const uint64_t x = X[w];
    pc += __popcll(x);
    if (x) one(w, x);
  }
  return s;
}

// The same digest with the work spread over the warp by bit position instead of by word
// (GD_DIG2): the warp walks the node's non-zero words (narrow: the ballot of y; wide: the rows of
// the occupancy bitmap) in lockstep, and lane l hashes bits l and l + 32 of each word, whose
// instance gids it holds in registers for the whole node (the columns are the module's).  The
// per-word row slot is one broadcast load; no lane loops over another lane's bits.
__device__ __forceinline__ unsigned long long digest_words2(const Dev& D, const NodeRec& R, uint64_t hn,
                                                            const uint64_t (&y)[DKW], int lane, uint32_t& pc) {
  const uint32_t logW = R.logW, L = R.L, B = R.B, W = 1u << logW;
  constexpr int OVQ = 8;                                   // columns held in registers: 256
  uint32_t ov[OVQ];                                        // instance gid of column 32 q + lane
#pragma unroll
  for (int q = 0; q < OVQ; ++q) {
    const uint32_t c = 32u * q + lane;
    ov[q] = ((uint32_t)q < 2 * W && c < R.n_cols) ? D.col_gid[R.col_off + c] : 0u;
  }
  auto col = [&](int q) -> uint32_t {                      // q >= OVQ (|Q| > 256): from L1
    const uint32_t c = 32u * q + lane;
    return c < R.n_cols ? D.col_gid[R.col_off + c] : 0u;
  };
  unsigned long long s = 0;
  auto slot_of = [&](uint32_t r) -> uint64_t {
    return r < L ? (uint64_t)(R.local_base + r) : (uint64_t)D.grow_gid[R.grow_off + r - L];
  };
  auto bits = [&](uint64_t hs, uint64_t x, uint32_t o0, uint32_t o1) {
    const bool b0 = (x >> lane) & 1ull, b1 = (x >> (lane + 32)) & 1ull;
    pc += (uint32_t)b0 + (uint32_t)b1;
    if (b0) s += mix64(hs ^ o0);
    if (b1) s += mix64(hs ^ o1);
  };
  const uint64_t* X = D.facts + R.off;
  if (logW >= 1) {                                         // wide block: occupied rows only
    const uint32_t rows = B >> logW, nocc = occ_words(rows);
    const uint64_t* OCC = X + occ_offset(B);
    for (uint32_t i = 0; i < nocc; ++i) {
      uint64_t ow = OCC[i];
      while (ow) {
        const uint32_t r = i * 64 + (__ffsll((long long)ow) - 1);
        ow &= ow - 1;
        const uint64_t hs = hn ^ (slot_of(r) << 32);
#pragma unroll
        for (int q = 0; q < MAXW; ++q) {
          if ((uint32_t)q >= W) break;
          const uint64_t x = X[((uint64_t)r << logW) + q];
          if (!x) continue;
          if (2 * q + 1 < OVQ) bits(hs, x, ov[2 * q], ov[2 * q + 1]);
          else bits(hs, x, col(2 * q), col(2 * q + 1));
        }
      }
    }
    return s;
  }
#pragma unroll
  for (int k = 0; k < DKW; ++k) {                          // narrow: one word per row
    unsigned m = __ballot_sync(FULL, y[k] != 0);
    while (m) {
      const int src = __ffs(m) - 1;
      m &= m - 1;
      const uint64_t x = shfl64(y[k], src);
      bits(hn ^ (slot_of((uint32_t)(src + 32 * k)) << 32), x, ov[0], ov[1]);
    }
  }
  for (uint32_t w0 = 32 * DKW; w0 < B; w0 += 32) {          // blocks beyond 128 words
    const uint64_t xl = w0 + lane < B ? X[w0 + lane] : 0ull;
    unsigned m = __ballot_sync(FULL, xl != 0);
    while (m) {
      const int src = __ffs(m) - 1;
      m &= m - 1;
      bits(hn ^ (slot_of(w0 + src) << 32), shfl64(xl, src), ov[0], ov[1]);
    }
  }
  return s;
}

// (a7) per-node digests d(n) = Σ mix64(mix64(n) ^ (slot<<32 | inst)) (C8).  A warp takes two
// nodes at a time: both NodeRecs, then the first 128 words of both blocks, are loaded before any
// bit is hashed (memory-level parallelism; the store is read once, coalesced).  A warp's nodes
// are nw apart, so consecutive ones almost always belong to the same app: the app sum is
// carried in a register and added once per app change.
__global__ void __launch_bounds__(256) k_digest(Dev D) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  unsigned long long app_sum = 0;
  uint32_t app_cur = 0xffffffffu;
  const uint32_t g0 = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  for (uint32_t n = g0; n < D.n_nodes; n += 2 * nw) {
    const uint32_t n2 = n + nw;
    const bool has2 = n2 < D.n_nodes;
    const NodeRec R = D.nodes[n];
    NodeRec R2 = R;
    if (has2) R2 = D.nodes[n2];
    const uint64_t hn = mix64((uint64_t)(n - D.app_node_base[R.app]));
    const uint64_t hn2 = has2 ? mix64((uint64_t)(n2 - D.app_node_base[R2.app])) : 0ull;
    uint64_t y[DKW], y2[DKW];
#pragma unroll
    for (int k = 0; k < DKW; ++k) {                         // (wide blocks read occupied rows instead)
      const uint32_t w = lane + 32 * k;
      y[k] = (R.logW == 0 && w < R.B) ? D.facts[R.off + w] : 0ull;
      y2[k] = (has2 && R2.logW == 0 && w < R2.B) ? D.facts[R2.off + w] : 0ull;
    }
    uint32_t pc = 0, pc2 = 0;                               // facts per node (readback sizes)
    const unsigned long long s = warp_sum64(GD_DIG2 ? digest_words2(D, R, hn, y, lane, pc)
                                                    : digest_words(D, R, hn, y, lane, pc));
    const unsigned long long s2 = !has2 ? 0ull : warp_sum64(GD_DIG2 ? digest_words2(D, R2, hn2, y2, lane, pc2)
                                                                    : digest_words(D, R2, hn2, y2, lane, pc2));
    pc = __reduce_add_sync(FULL, pc);
    pc2 = __reduce_add_sync(FULL, pc2);
    if (lane == 0) {
      D.node_digest[n] = s;
      D.node_popc[n] = pc;
      if (has2) { D.node_digest[n2] = s2; D.node_popc[n2] = pc2; }
      if (R.app != app_cur) {
        if (app_sum) atomicAdd(&D.app_digest[app_cur], app_sum);
        app_cur = R.app;
        app_sum = 0;
      }
      app_sum += s;
      if (has2) {
        if (R2.app != app_cur) {
          if (app_sum) atomicAdd(&D.app_digest[app_cur], app_sum);
          app_cur = R2.app;
          app_sum = 0;
        }
        app_sum += s2;
      }
    }
  }
  if (lane == 0 && app_sum) atomicAdd(&D.app_digest[app_cur], app_sum);
}

// Readback kernels over nodes n0 .. n1-1, or over list[0 .. n1-n0) when list != nullptr.
__global__ void k_popc(Dev D, uint32_t n0, uint32_t n1, uint64_t* out, const uint32_t* list) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n1 - n0; i += nw) {
    const uint32_t n = list ? list[i] : n0 + i;
    const NodeRec R = D.nodes[n];
    unsigned long long c = 0;
    for (uint32_t w = lane; w < R.B; w += 32) c += __popcll(D.facts[R.off + w]);
    c = warp_sum64(c);
    if (lane == 0) out[i] = c;
  }
}

// bits of IN(n) -> ascending (slot gid << 32 | inst gid): row-major order is ascending because
// rows are locals < statics < heap in gid order and columns are sorted instance gids.
__global__ void k_expand(Dev D, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs,
                         const uint32_t* list) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n1 - n0; i += nw) {
    const uint32_t n = list ? list[i] : n0 + i;
    const NodeRec R = D.nodes[n];
    const uint32_t local_base = R.local_base;
    const uint32_t logW = R.logW, L = R.L, B = R.B;
    uint64_t base = ptr[i];
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
        const uint64_t slot = r < L ? (uint64_t)(local_base + r) : (uint64_t)D.grow_gid[R.grow_off + r - L];
        while (x) {
          const int b = __ffsll((long long)x) - 1;
          x &= x - 1;
          pairs[pos++] = (slot << 32) | D.col_gid[R.col_off + j * 64 + b];
        }
      }
      base += __shfl_sync(FULL, incl, 31);
    }
  }
}

// Exclusive prefix of u32 counts into u64 offsets: per-block scan of SCAN_ITEMS elements (block
// totals to tmp), one-block scan of the totals, then each block adds its offset.
constexpr uint32_t SCAN_T = 1024, SCAN_PER = 8, SCAN_ITEMS = SCAN_T * SCAN_PER;
__device__ __forceinline__ unsigned long long block_exclusive_scan(unsigned long long v, unsigned long long* total) {
  __shared__ unsigned long long ws[32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) { const unsigned long long t = __shfl_up_sync(FULL, x, o); if (lane >= o) x += t; }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  if (w == 0) {
    unsigned long long z = lane < (int)(blockDim.x >> 5) ? ws[lane] : 0ull;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) { const unsigned long long t = __shfl_up_sync(FULL, z, o); if (lane >= o) z += t; }
    ws[lane] = z;
  }
  __syncthreads();
  const unsigned long long incl = x + (w ? ws[w - 1] : 0ull);
  *total = ws[(blockDim.x >> 5) - 1];
  __syncthreads();
  return incl - v;
}
__global__ void __launch_bounds__(SCAN_T) k_scan_blocks(const uint32_t* c, uint32_t n, uint64_t* ptr, uint64_t* tot) {
  const uint64_t b0 = (uint64_t)blockIdx.x * SCAN_ITEMS + (uint64_t)threadIdx.x * SCAN_PER;
  uint32_t v[SCAN_PER];
  unsigned long long sum = 0;
#pragma unroll
  for (int i = 0; i < (int)SCAN_PER; ++i) { v[i] = b0 + i < n ? c[b0 + i] : 0u; sum += v[i]; }
  unsigned long long total;
  unsigned long long run = block_exclusive_scan(sum, &total);
#pragma unroll
  for (int i = 0; i < (int)SCAN_PER; ++i) { if (b0 + i < n) ptr[b0 + i] = run; run += v[i]; }
  if (threadIdx.x == 0) tot[blockIdx.x] = total;
}
__global__ void __launch_bounds__(SCAN_T) k_scan_totals(uint64_t* tot, uint32_t nb, uint64_t* ptr, uint32_t n) {
  unsigned long long carry = 0;
  for (uint32_t b = 0; b < nb; b += SCAN_T) {
    const uint32_t i = b + threadIdx.x;
    const unsigned long long v = i < nb ? tot[i] : 0ull;
    unsigned long long total;
    const unsigned long long ex = block_exclusive_scan(v, &total);
    if (i < nb) tot[i] = carry + ex;
    carry += total;
  }
  if (threadIdx.x == 0) ptr[n] = carry;
}
__global__ void __launch_bounds__(SCAN_T) k_scan_add(uint64_t* ptr, uint32_t n, const uint64_t* tot) {
  const uint64_t b0 = (uint64_t)blockIdx.x * SCAN_ITEMS;
  const unsigned long long add = tot[blockIdx.x];
  for (uint32_t i = threadIdx.x; i < SCAN_ITEMS; i += SCAN_T)
    if (b0 + i < n) ptr[b0 + i] += add;
}

}  // namespace

size_t scan_tmp_words(uint32_t n) { return (size_t)((n + SCAN_ITEMS - 1) / SCAN_ITEMS) + 1; }

cudaError_t launch_scan_counts(const uint32_t* counts, uint32_t n, uint64_t* ptr, uint64_t* tmp, cudaStream_t s) {
  const uint32_t nb = (n + SCAN_ITEMS - 1) / SCAN_ITEMS;
  if (nb) k_scan_blocks<<<nb, SCAN_T, 0, s>>>(counts, n, ptr, tmp);
  k_scan_totals<<<1, SCAN_T, 0, s>>>(tmp, nb, ptr, n);
  if (nb) k_scan_add<<<nb, SCAN_T, 0, s>>>(ptr, n, tmp);
  return cudaGetLastError();
}

cudaError_t launch_rebase(const Dev& D, NodeRec* nodes, uint32_t* nodemeth, uint32_t* rowptr, uint32_t* argptr,
                          const AppBase* bases, cudaStream_t s) {
  uint32_t blocks = (D.n_nodes + 255) / 256;
  blocks = blocks == 0 ? 1u : (blocks > 148 * 8 ? 148 * 8 : blocks);
  k_rebase<<<blocks, 256, 0, s>>>(D, nodes, nodemeth, rowptr, argptr, bases);
  return cudaGetLastError();
}

cudaError_t launch_edges(const Dev& D, Edge* edges, InlEdge* inl, NodeRec* nodes, const uint32_t* ecol,
                         const uint8_t* ekind, const uint32_t* exoff, cudaStream_t s) {
  uint32_t blocks = (D.n_nodes + 255) / 256;
  blocks = blocks == 0 ? 1u : (blocks > 148 * 8 ? 148 * 8 : blocks);
  k_edges<<<blocks, 256, 0, s>>>(D, edges, inl, nodes, ecol, ekind, exoff);
  return cudaGetLastError();
}

cudaError_t launch_nmask_rebuild(const Dev& D, cudaStream_t s) {
  k_nmask_rebuild<<<1184, 256, 0, s>>>(D);
  return cudaGetLastError();
}

cudaError_t launch_seed(const Dev& D, cudaStream_t s) {
  if (D.n_seed_pairs) k_apply_seeds<<<(D.n_seed_pairs + 255) / 256, 256, 0, s>>>(D);
  k_seed<<<1, 32, 0, s>>>(D);
  return cudaGetLastError();
}

// Instantiations: narrow batches (WIDE = false) and wide batches by the widest row of the
// batch (MW = 2, 4, 8 words: register arrays sized to it), each with and without the
// byte-model counters (CNT).  Large narrow batches (Dev::hiocc) use a 4-CTA/SM build (64
// registers): their big rounds are item-throughput bound and gain from the extra warps, while
// small batches are round-latency bound and lose to its spills.
template <bool CNT>
static const void* fixpoint_fn(uint32_t wide, uint32_t hiocc) {
  switch (wide) {
    case 0: return hiocc ? (const void*)k_fixpoint<false, CNT, 1, GD_MINB_HI>
                         : (const void*)k_fixpoint<false, CNT, 1, GD_MINB>;
    case 1: return (const void*)k_fixpoint<true, CNT, 2, GD_MINB_WIDE>;
    case 2: return (const void*)k_fixpoint<true, CNT, 4, GD_MINB_WIDE>;
    default: return (const void*)k_fixpoint<true, CNT, 8, GD_MINB_WIDE>;
  }
}

int fixpoint_max_blocks(int device, uint32_t wide, uint32_t hiocc) {
  int sms = 0, occ = 0, occ2 = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fixpoint_fn<true>(wide, hiocc), THREADS, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, fixpoint_fn<false>(wide, hiocc), THREADS, 0);
  occ = occ2 < occ ? occ2 : occ;          // one grid size serves both instantiations
  return sms * (occ > 0 ? occ : 1);
}

cudaError_t launch_fixpoint(const Dev& D, uint32_t blocks, cudaStream_t s) {
  Dev d = D;
  void* args[] = {&d};
  const void* f = D.count ? fixpoint_fn<true>(D.wide, D.hiocc) : fixpoint_fn<false>(D.wide, D.hiocc);
  return cudaLaunchCooperativeKernel(f, dim3(blocks), dim3(THREADS), args, 0, s);
}

template <bool CNT>
static const void* sbda_fn(uint32_t wide) {
  switch (wide) {
    case 0: return (const void*)k_sbda<false, CNT, 1>;
    case 1: return (const void*)k_sbda<true, CNT, 2>;
    case 2: return (const void*)k_sbda<true, CNT, 4>;
    default: return (const void*)k_sbda<true, CNT, 8>;
  }
}

int sbda_max_blocks(int device, uint32_t wide) {
  int sms = 0, occ = 0, occ2 = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sbda_fn<true>(wide), THREADS, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, sbda_fn<false>(wide), THREADS, 0);
  occ = occ2 < occ ? occ2 : occ;
  return sms * (occ > 0 ? occ : 1);
}

cudaError_t launch_sbda(const Dev& D, uint32_t blocks, cudaStream_t s) {
  Dev d = D;
  void* args[] = {&d};
  return cudaLaunchCooperativeKernel(D.count ? sbda_fn<true>(D.wide) : sbda_fn<false>(D.wide), dim3(blocks),
                                     dim3(THREADS), args, 0, s);
}

cudaError_t launch_meth_csr(const Dev& D, uint32_t* ptr, uint32_t* nodes, uint32_t* cursor, cudaStream_t s) {
  cudaMemsetAsync(ptr, 0, (size_t)(D.n_meths + 1) * 4, s);
  cudaMemsetAsync(cursor, 0, (size_t)D.n_meths * 4, s);
  k_meth_count<<<1184, 256, 0, s>>>(D, ptr);
  k_meth_scan<<<1, 1024, 0, s>>>(ptr, D.n_meths);
  k_meth_fill<<<1184, 256, 0, s>>>(D, ptr, cursor, nodes);
  return cudaGetLastError();
}

template <bool CNT>
static void round_launch(const Dev& D, uint32_t round, uint32_t blocks, cudaStream_t s) {
  switch (D.wide) {
    case 0: k_round<false, CNT, 1><<<blocks, THREADS, 0, s>>>(D, round); break;
    case 1: k_round<true, CNT, 2><<<blocks, THREADS, 0, s>>>(D, round); break;
    case 2: k_round<true, CNT, 4><<<blocks, THREADS, 0, s>>>(D, round); break;
    default: k_round<true, CNT, 8><<<blocks, THREADS, 0, s>>>(D, round); break;
  }
}

cudaError_t launch_round(const Dev& D, uint32_t round, uint32_t blocks, cudaStream_t s) {
  if (D.count) round_launch<true>(D, round, blocks, s);
  else round_launch<false>(D, round, blocks, s);
  return cudaGetLastError();
}

static uint32_t grid_for(uint32_t items) {
  uint32_t blocks = (items + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  return blocks ? blocks : 1;
}

cudaError_t launch_digest(const Dev& D, cudaStream_t s) {
  k_digest<<<grid_for(D.n_nodes), 256, 0, s>>>(D);
  return cudaGetLastError();
}

cudaError_t launch_popc(const Dev& D, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s, const uint32_t* list) {
  k_popc<<<grid_for(n1 - n0), 256, 0, s>>>(D, n0, n1, out, list);
  return cudaGetLastError();
}

cudaError_t launch_expand(const Dev& D, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs,
                          cudaStream_t s, const uint32_t* list, uint32_t max_blocks) {
  uint32_t g = grid_for(n1 - n0);
  if (max_blocks && g > max_blocks) g = max_blocks;
  k_expand<<<g, 256, 0, s>>>(D, n0, n1, ptr, pairs, list);
  return cudaGetLastError();
}

}  // namespace gd
