python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q --durations=3 2>&1 | tail -5
for c in c3 c5 c1 c2 c4; do timeout 900 python bench.py --workload $c --steps 10 --warmup 3 > gpurun_out/bench6_$c.json 2> gpurun_out/bench6_$c.err; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches6_c5.csv python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_lane -s 3 -c 1 -o gpurun_out/full6_c5 python bench.py --workload c5 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu6_c5.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches6_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_step -s 3 -c 1 -o gpurun_out/full6_c3 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu6_c3.log 2>&1
for f in gpurun_out/bench6_*.err; do tail -n 2 $f; done
