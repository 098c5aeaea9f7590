# experiment: does the grid-barrier flag placement explain the per-instance C3 bimodality?
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for sh in 0 4 64 1024 4096 16384; do echo "shift ${sh}KB"; GEM_EXP_BAR_SHIFT_KB=$sh PYTHONPATH=. python scripts/bimodal.py 2>&1 | tail -4 | awk '{print $2, $5, $6}'; done
