mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python scripts/prof_run.py --cfg c5 --cycles 20 --streams 4096 --phases 2>&1 | grep -v "^{" | tail -8
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gem_lane -s 1 -c 1 -o gpurun_out/full_c5 python scripts/prof_run.py --cfg c5 --cycles 10 --streams 4096 > gpurun_out/ncu_c5.log 2>&1
ncu -i gpurun_out/full_c5.ncu-rep --page source --csv --print-source sass > gpurun_out/c5_sass.csv 2>/dev/null; wc -l gpurun_out/c5_sass.csv
