# one iteration: build, gpu tests, fine + phase profile of c1/c3, c5 lane kernel rate
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python scripts/fine_prof.py c1 c3 2>&1 | tail -30
for c in c1 c2 c3; do timeout 300 python scripts/prof_run.py --cfg $c --cycles 1000 2>&1 | grep -v "n_pi"; done
timeout 300 python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1"
timeout 300 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1
