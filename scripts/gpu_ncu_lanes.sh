python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
ncu --set full --clock-control none --import-source on -k regex:gem_lane -s 1 -c 1 -o gpurun_out/prof_c5_lanes python scripts/prof_run.py --cfg c5 --cycles 4 --streams 4096 > gpurun_out/ncu_c5.log 2>&1
tail -3 gpurun_out/ncu_c5.log
