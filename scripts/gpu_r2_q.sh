python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python scripts/readback_bench.py
