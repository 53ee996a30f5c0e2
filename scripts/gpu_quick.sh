# quick GPU check: build, parity tests, median + corpus bench lines
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 600 python bench.py --workload median --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1
timeout 900 python bench.py --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1
