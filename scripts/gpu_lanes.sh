python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu.py -x -q -k "c5" 2>&1 | tail -3
for g in 1 2 4; do GEM_LANE_GROUPS=$g python scripts/prof_run.py --cfg c5 --cycles 50 --streams 4096 2>&1 | grep "launch 1"; done
python scripts/prof_run.py --cfg c5 --cycles 50 --streams 4096 2>&1 | tail -1 | cut -c1-500
