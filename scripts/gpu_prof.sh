set -x
python -c "import __graft_entry__ as g; g.build()"
python scripts/prof_run.py --cfg c1 --cycles 2000
python scripts/prof_run.py --cfg c3 --cycles 2000
python scripts/prof_run.py --cfg c2 --cycles 2000
ncu --set full --clock-control none --import-source on -k regex:gem_step -s 1 -c 1 -o gpurun_out/prof_c1 python scripts/prof_run.py --cfg c1 --cycles 200 > gpurun_out/ncu_c1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:gem_step -s 1 -c 1 -o gpurun_out/prof_c3 python scripts/prof_run.py --cfg c3 --cycles 30 > gpurun_out/ncu_c3.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
tail -2 gpurun_out/ncu_c1.log gpurun_out/ncu_c3.log
