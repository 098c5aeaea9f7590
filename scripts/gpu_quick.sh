python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in c1 c3; do timeout 300 python scripts/prof_run.py --cfg $c --cycles 1000 --phases 2>&1 | grep -v "n_pi"; done
