python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for b in 1 2 3; do echo "bps=$b"; GEM_BPS=$b timeout 600 python scripts/prof_run.py --cfg c4 --cycles 100 2>&1 | grep "launch 1\|Error\|error"; done
