python -c "import __graft_entry__ as g; g.build()" > gpurun_out/w_build.log 2>&1 || { tail -20 gpurun_out/w_build.log; exit 1; }
for c in c3 c1; do
O=$(python -c "from tests.common import MAP_OPTS; print(MAP_OPTS['$c'] + ' words=1')")
timeout 300 python scripts/prof_run.py --cfg $c --phases --map-opts "$O" 2>&1 | grep -v "^{" | tail -6
done
