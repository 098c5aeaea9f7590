mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "levels=10 key=2" "levels=10 key=2 part_size=3000" "levels=10 key=2 part_size=2500" "levels=10 key=2 part_size=3200"; do
  echo "== $o"; timeout 600 python scripts/prof_run.py --cfg c2 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|Error" | cut -c1-200
done
