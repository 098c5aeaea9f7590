mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do timeout 600 python scripts/prof_run.py --cfg c5 --cycles 100 --streams 4096 --phases 2>&1 | grep "launch 1\|lane phases\|rror" | cut -c1-230; done
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
