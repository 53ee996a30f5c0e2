# round-2 probe: box hardware, build, GPU parity tests except the stored full-size fixtures
set -x
nproc; lscpu | grep -E "Model name|^CPU\(s\)|Socket|Thread"; free -g; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py -k "not hybrid_schedule" 2>&1 | tail -8
