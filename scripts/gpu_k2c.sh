mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep "launch 1\|lane phases\|Error" | cut -c1-250
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python bench.py --workload c5 --steps 5 --warmup 3 > gpurun_out/b_c5.json 2>gpurun_out/b_c5.err; python -c "import json; d=json.loads(open('gpurun_out/b_c5.json').read().strip().splitlines()[-1]); print('c5', round(d['value']), round(d['e2e']['value']), d['roofline']['frac'])"
