#!/bin/bash
# Per-kernel durations of the device layout (ncu launch list, serialised) on a 60-app batch and the
# worst preset, plus per-round traces of small / chain (light-round floor).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/lp_build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_dl_ --csv \
  --log-file gpurun_out/lp_launches.csv python scripts/load_timing.py 60 > gpurun_out/lp_ncu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_dl_ --csv \
  --log-file gpurun_out/lp_launches_worst.csv python scripts/load_timing.py app:$(python -c "
from synth import generator as G; print([i for i in range(1000) if G.corpus_config(i).q_cap > 64][0])") > gpurun_out/lp_ncu_worst.log 2>&1
timeout 300 python scripts/trace_rounds.py small > gpurun_out/lp_trace_small.log 2>&1
timeout 300 python scripts/trace_rounds.py chain > gpurun_out/lp_trace_chain.log 2>&1
