python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 1200 python -m pytest tests -m gpu -x -q --durations=5 2>&1 | tail -15
python scripts/prof_run.py --cfg c3 --cycles 1000 --phases 2>&1 | grep -v "n_pi"
python scripts/prof_run.py --cfg c4 --cycles 200 2>&1 | tail -3
python scripts/prof_run.py --cfg c5 --cycles 20 --streams 4096 2>&1 | tail -3
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err; cut -c1-400 gpurun_out/bench.json
