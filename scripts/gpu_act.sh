mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k activity > gpurun_out/pytest_act.log 2>&1; tail -3 gpurun_out/pytest_act.log
timeout 900 python scripts/activity_bench.py --cycles 2000 > gpurun_out/activity.jsonl 2> gpurun_out/activity.err; cat gpurun_out/activity.jsonl; tail -3 gpurun_out/activity.err
