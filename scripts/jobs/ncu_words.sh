python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in c1 c3; do
O=$(python -c "from tests.common import MAP_OPTS; print(MAP_OPTS['$c'] + ' words=1')")
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gem_word_kernel -s 1 -c 1 -f -o gpurun_out/w_ncu_$c python scripts/prof_run.py --cfg $c --cycles 200 --map-opts "$O" > gpurun_out/w_ncu_$c.log 2>&1
tail -2 gpurun_out/w_ncu_$c.log
done
