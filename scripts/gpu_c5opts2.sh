mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
M="refine=0 lanes=1 key=2 merge_cap=60000 lane_words=14000"
for o in "$M" "$M levels=10" "$M levels=11" "$M levels=12"; do
  echo "== $o"; timeout 900 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases --map-opts "$o" 2>&1 | grep "launch 1\|lane phases\|Error" | cut -c1-230
done
timeout 900 python bench.py --steps 5 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c3', d['value'], d['cpu_baseline']['value'], d['cpu_baseline_mt'])"
