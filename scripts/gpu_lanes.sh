python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for cfg in "2 1" "2 2" "1 1" "1 2" "1 4"; do set -- $cfg; echo "bps=$1 groups=$2"; GEM_LANE_BPS=$1 GEM_LANE_GROUPS=$2 timeout 300 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), d['config']['stream_group'], d['config']['grid'], d['roofline']['kernel_ms_per_step'])"; done
