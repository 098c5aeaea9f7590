python -c "import __graft_entry__ as g; g.build()"
for c in c1 c2 c3; do python scripts/prof_run.py --cfg $c --cycles 1000 --phases 2>&1 | grep -v "n_pi"; done
