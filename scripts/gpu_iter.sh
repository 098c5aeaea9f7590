# one iteration: build, gpu tests, phase profile of c1/c2/c3, c4 and c5 rates, c3 partitioning variants
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for c in c1 c2 c3; do timeout 300 python scripts/prof_run.py --cfg $c --cycles 1000 --phases 2>&1 | grep -v "n_pi"; done
timeout 300 python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1"
timeout 300 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-200
for o in "part_size=4000 max_parts=296" "part_size=3000 max_parts=444"; do for b in 2 3; do echo "== $o bps=$b"; GEM_BPS=$b timeout 300 python scripts/prof_run.py --cfg c3 --cycles 1000 --map-opts "$o" 2>&1 | grep "launch 1\|resident"; done; done
