mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "dataflow" 2>&1 | tail -3
EXP_CFG="c3 c2" bash scripts/gpu_ab.sh 2>&1 | grep -v "gread split"
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
