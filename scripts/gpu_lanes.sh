python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu.py -x -q -k "c5" 2>&1 | tail -2
python scripts/prof_run.py --cfg c5 --cycles 50 --streams 4096 2>&1 | grep "launch 1\|n_pi" | cut -c1-400
GEM_LANE_BPS=1 python scripts/prof_run.py --cfg c5 --cycles 50 --streams 4096 2>&1 | grep "launch 1"
