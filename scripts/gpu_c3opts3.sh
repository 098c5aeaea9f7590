mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "part_size=8000 max_parts=148 levels=10 key=2" "part_size=10000 max_parts=148 levels=10 key=2" "part_size=12000 max_parts=148 levels=10 key=2" "part_size=16000 max_parts=148 levels=10 key=2" "part_size=20000 max_parts=148 levels=10 key=2" "part_size=8000 max_parts=148 levels=10 key=2 refine=0"; do
  echo "== $o"; timeout 600 python scripts/prof_run.py --cfg c3 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|Error" | cut -c1-200
done
