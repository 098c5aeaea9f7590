mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "stages=1 levels=10 key=2 part_size=18000" "stages=1 levels=10 key=2 part_size=22000" "stages=1 levels=10 key=2 part_size=24000" "stages=1 levels=10 key=2 part_size=20000 max_parts=300"; do
  echo "== $o"; timeout 900 python scripts/prof_run.py --cfg c4 --cycles 100 --map-opts "$o" 2>&1 | grep "launch 1\|rror"
done
