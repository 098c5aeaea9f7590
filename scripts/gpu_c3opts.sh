mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "part_size=8000 max_parts=148 levels=10 key=2" "part_size=8000 max_parts=148 levels=11 key=2" "part_size=8000 max_parts=148 levels=13 key=2" "part_size=6000 max_parts=148 levels=10 key=2" "part_size=8000 max_parts=148 levels=10 key=2 leafcap=256"; do
  echo "== $o"; timeout 600 python scripts/prof_run.py --cfg c3 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|Error" | cut -c1-200
done
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
