python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for o in "part_size=8000 max_parts=148 banks=0" "part_size=8000 max_parts=148" "part_size=8000 max_parts=148 levels=10" "part_size=8000 max_parts=148 levels=11"; do
  echo "== $o"; timeout 300 python scripts/prof_run.py --cfg c3 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep -v n_pi
done
