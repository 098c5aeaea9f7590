python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for o in "refine=0 lanes=1 part_size=12000" "refine=0 lanes=1 part_size=20000" "refine=0 lanes=1 part_size=30000"; do
  echo "== $o"; timeout 600 python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu-baseline --map-opts "$o" 2>&1 | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); c=d['config']; print(round(d['value']), c['parts'], c['stream_group'], d['roofline']['frac'])"
done
