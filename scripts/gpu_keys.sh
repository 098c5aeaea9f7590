python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for o in "part_size=8000 max_parts=148 levels=10" "part_size=8000 max_parts=148 levels=10 key=2" "part_size=8000 max_parts=148 levels=10 key=2 merge_cap=40000" "part_size=4000 max_parts=148 levels=10 key=2"; do
  echo "== c3 $o"; timeout 300 python scripts/prof_run.py --cfg c3 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]"
done
for o in "refine=0 lanes=1 key=2" "refine=0 lanes=1 key=2 merge_cap=60000" "refine=0 lanes=1 key=2 merge_cap=60000 part_size=12000"; do
  echo "== c5 $o"; timeout 600 python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu-baseline --map-opts "$o" 2>&1 | tail -1 | cut -c1-200
done
