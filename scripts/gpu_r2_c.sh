python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_ooc.py tests/test_gpu_parity.py tests/test_gpu_corpus.py -x -q 2>&1 | tail -15
