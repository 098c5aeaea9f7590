python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python scripts/prof_run.py --cfg c1 --cycles 1000 --phases 2>&1 | grep "launch 1\|critical CTA [0-9]"
for o in "part_size=8000 max_parts=148" "part_size=8000 max_parts=148 levels=10"; do
  echo "== $o"; timeout 300 python scripts/prof_run.py --cfg c3 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|all CTAs"
done
for o in "" "levels=10"; do
  echo "== c2 $o"; timeout 300 python scripts/prof_run.py --cfg c2 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]"
done
