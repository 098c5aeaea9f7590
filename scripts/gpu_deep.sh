mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
EXP_CFG="c3 c1 c2" bash scripts/gpu_ab.sh 2>&1 | grep "==\|launch 1\|critical CTA [0-9]"
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
