mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
M="refine=0 lanes=1 key=2 merge_cap=60000 lane_words=14000 levels=10"
for o in "$M" "$M merge_ratio=0.4" "$M merge_ratio=0.5"; do
  echo "== $o"; timeout 900 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --map-opts "$o" 2>&1 | grep "launch 1\|rror" | cut -c1-200
done
