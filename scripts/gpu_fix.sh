mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
EXP_CFG="c1 c3" bash scripts/gpu_ab.sh 2>&1 | grep -v "gread split"
timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep "launch 1\|lane phases\|Error" | cut -c1-250
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
