python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for w in c1 c3; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench_$w.json; done
timeout 600 python bench.py --workload c5 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench_c5.json
