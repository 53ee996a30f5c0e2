# A/B on one box: the committed baseline kernel (.ab/, built into a separate .so) vs the tree's
# variants.  usage: bash scripts/gpu_ab.sh "<flags>" ...
set -e
python -c "import __graft_entry__ as g; g.build()"
mkdir -p /tmp/abbase/x/csrc /tmp/abbase/include
cp .ab/kernels_base.cu /tmp/abbase/x/csrc/kernels.cu; cp .ab/loader_base.cu /tmp/abbase/x/csrc/loader.cu
cp .ab/internal_base.cuh /tmp/abbase/x/csrc/internal.cuh; cp include/gdroid.h /tmp/abbase/include/
git_hdr=$(ls .ab/gdroid_base.h 2>/dev/null || true); [ -n "$git_hdr" ] && cp .ab/gdroid_base.h /tmp/abbase/include/gdroid.h
cp paper_conf_ipps_yuwobby20_b200/libgdroid.so /tmp/lib_tree.so
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -shared -Xcompiler -fPIC -I /tmp/abbase/include \
  -o /tmp/lib_base.so /tmp/abbase/x/csrc/loader.cu /tmp/abbase/x/csrc/kernels.cu
for rep in 1 2; do
  cp /tmp/lib_base.so paper_conf_ipps_yuwobby20_b200/libgdroid.so; touch paper_conf_ipps_yuwobby20_b200/libgdroid.so
  for w in ${WORKLOADS:-small median corpus}; do echo "== base $w"; timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['rounds_per_step'])"; done
  for v in "$@"; do
    GDROID_NVCC_FLAGS="-DGD_AB $v" python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build()"
    for w in ${WORKLOADS:-small median corpus}; do echo "== [$v] $w"; timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['rounds_per_step'])"; done
  done
done
