mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
M="refine=0 lanes=1 key=2 merge_cap=60000 lane_words=14000 levels=10"
for o in "$M lane_banks=0" "$M" "$M lane_banks=0" "$M"; do
  echo "== $o"; timeout 900 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases --map-opts "$o" 2>&1 | grep "launch 1\|lane phases\|Error" | cut -c1-230
done
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
