python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in c1 c3; do python scripts/prof_run.py --cfg $c --cycles 1000 --phases 2>&1 | grep -v "n_pi"; done
python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1"
