python -c "import __graft_entry__ as g; g.build()"
ncu --set full --clock-control none --import-source on -k regex:gem_step -s 1 -c 1 -o gpurun_out/prof_c1 python scripts/prof_run.py --cfg c1 --cycles 300 > gpurun_out/ncu_c1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:gem_step -s 1 -c 1 -o gpurun_out/prof_c3 python scripts/prof_run.py --cfg c3 --cycles 40 > gpurun_out/ncu_c3.log 2>&1
tail -2 gpurun_out/ncu_c1.log gpurun_out/ncu_c3.log
