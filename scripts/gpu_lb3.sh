mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
echo "== base (K=2, 2 CTAs/SM)"; GEM_EXP_LIB=$PWD/exp_libs/libgem_base.so timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 2>&1 | grep "launch 1\|rror"
echo "== base K=1"; GEM_LANE_GROUPS=1 GEM_EXP_LIB=$PWD/exp_libs/libgem_base.so timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 2>&1 | grep "launch 1\|rror"
echo "== lb3 K=1 3 CTAs/SM"; GEM_LANE_GROUPS=1 GEM_LANE_BPS=3 GEM_EXP_LIB=$PWD/exp_libs/libgem_lb3.so timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 2>&1 | grep "launch 1\|rror"
