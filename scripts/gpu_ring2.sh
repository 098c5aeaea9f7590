mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
EXP_CFG="c3" bash scripts/gpu_ab.sh 2>&1 | grep -v "gread split"
timeout 600 python bench.py --workload c4 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4', d['value'], d['roofline']['frac'])"
