mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in "" 1 2 4; do echo "== run=$r"; GEM_LANE_RUN=$r timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep "launch 1\|lane phases\|Error" | cut -c1-250; done
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python bench.py --workload c5 --steps 5 --warmup 3 > gpurun_out/b_c5.json 2>gpurun_out/b_c5.err; tail -c 600 gpurun_out/b_c5.json
