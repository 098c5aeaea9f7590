mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for f in 0 0.3 0.47 0.7 0.9; do echo "== frac $f"; GEM_L2_FRAC=$f timeout 900 python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1\|rror"; done
echo "== default"; timeout 900 python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1\|rror"
EXP_CFG="c3" bash scripts/gpu_ab.sh 2>&1 | grep "==\|launch 1"
