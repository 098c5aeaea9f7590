mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b_c5.json 2>gpurun_out/b_c5.err; python -c "import json; d=json.loads(open('gpurun_out/b_c5.json').read().strip().splitlines()[-1]); print('c5', round(d['value']), d['config']['grid'], d['roofline']['kernel_ms_per_step'], d['roofline']['frac'])"
timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep "lane phases"
