python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for w in chain median corpus8 small; do timeout 300 python scripts/trace_rounds.py $w; done
