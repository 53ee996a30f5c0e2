# round 2: parity tests of the new paths + first corpus1000 bench lines (reduced app counts)
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py::test_corpus_digest_all --deselect tests/test_gpu_fullsize.py::test_corpus_wide_apps -k "not preset_full_size or small or median" 2>&1 | tail -8
timeout 900 python bench.py --n-apps 100 --steps 2 --warmup 1 --no-per-config 2>&1 | tail -3
timeout 900 python bench.py --workload corpus8 --steps 5 --warmup 2 --no-cpu-baseline --e2e-readback digests 2>&1 | tail -3
