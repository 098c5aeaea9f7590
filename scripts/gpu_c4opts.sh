mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "stages=2 levels=10 key=2 part_size=16000" "stages=2 levels=10 key=2 part_size=18000" "stages=2 levels=10 key=2 part_size=22000" "stages=2 levels=10 key=2 part_size=25000" "stages=2 levels=10 key=2 part_size=20000 max_parts=400"; do
  echo "== $o"; timeout 900 python scripts/prof_run.py --cfg c4 --cycles 100 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|all CTAs\|Error\|rror" | cut -c1-220
done
