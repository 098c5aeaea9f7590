mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -1
timeout 900 python bench.py --workload c4 --steps 10 --warmup 3 > gpurun_out/bench15_c4.json 2> gpurun_out/bench15_c4.err; tail -c 300 gpurun_out/bench15_c4.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches15_c4.csv python bench.py --workload c4 --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_step -s 3 -c 1 -o gpurun_out/full15_c4 python bench.py --workload c4 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu15_c4.log 2>&1
ls -la gpurun_out/full15_c4.ncu-rep
