mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
M="refine=0 lanes=1 key=2 merge_cap=60000"
run() { echo "== $1 | $2 | $3"; env $3 GEM_EXP_LIB=$PWD/exp_libs/$1 timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases --map-opts "$2" 2>&1 | grep "launch 1\|lane phases\|Error\|error" | cut -c1-250; }
run libgem_ring.so "$M" ""
run libgem_noring.so "$M" ""
run libgem_noring.so "$M lane_words=14000" ""
run libgem_noring.so "$M lane_words=14000" "GEM_LANE_GROUPS=1"
run libgem_noring.so "$M lane_words=13000" ""
timeout 900 python -m pytest tests -m gpu -x -q -k "c5 or lane" 2>&1 | tail -2
