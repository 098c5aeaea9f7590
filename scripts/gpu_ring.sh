mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
EXP_CFG="c1 c3 c2" bash scripts/gpu_ab.sh 2>&1 | grep -v "gread split"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
