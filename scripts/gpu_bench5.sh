python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in c3 c1 c2 c4 c5; do timeout 900 python bench.py --workload $c --steps 10 --warmup 3 > gpurun_out/bench5_$c.json 2> gpurun_out/bench5_$c.err; done
timeout 600 python bench.py --workload c4 --steps 5 --warmup 3 --map-opts "stages=2 levels=10" --no-cpu-baseline > gpurun_out/bench5_c4l10.json 2>&1
tail -2 gpurun_out/bench5_*.err
