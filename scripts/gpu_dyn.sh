mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "c5 or lane" > gpurun_out/pytest_lane.log 2>&1; tail -2 gpurun_out/pytest_lane.log
for d in 1 0; do GEM_LANE_DYN=$d timeout 600 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b_dyn$d.json 2>gpurun_out/b_dyn$d.err; python -c "import json; d=json.loads(open('gpurun_out/b_dyn$d.json').read().strip().splitlines()[-1]); print('dyn=$d', round(d['value']), d['config']['grid'], d['roofline']['kernel_ms_per_step'])"; done
timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep -v "^{" | tail -4
