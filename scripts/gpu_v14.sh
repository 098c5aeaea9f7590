# round-1 measurement v14: smoke, GPU tests, bench lines C1-C5 + reference arm, ncu launch lists and full captures (C3, C5)
mkdir -p gpurun_out
nproc; grep -m1 "model name" /proc/cpuinfo
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q --durations=3 > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
for c in c3 c5 c1 c2 c4; do timeout 900 python bench.py --workload $c --steps 10 --warmup 3 > gpurun_out/bench14_$c.json 2> gpurun_out/bench14_$c.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench14_ref.json 2> gpurun_out/bench14_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches14_c5.csv python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_lane -s 3 -c 1 -o gpurun_out/full14_c5 python bench.py --workload c5 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu14_c5.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches14_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_step -s 3 -c 1 -o gpurun_out/full14_c3 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu14_c3.log 2>&1
ncu -i gpurun_out/full14_c5.ncu-rep --page source --csv --print-source sass > gpurun_out/c5_sass14.csv 2>/dev/null
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches14_c4.csv python bench.py --workload c4 --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_step -s 3 -c 1 -o gpurun_out/full14_c4 python bench.py --workload c4 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu14_c4.log 2>&1
for f in gpurun_out/bench14_*.err; do tail -n 1 $f; done
