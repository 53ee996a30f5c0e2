python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python scripts/e2e_diag.py 200
GDROID_HOST_THREADS=8 timeout 900 python scripts/e2e_diag.py 200
