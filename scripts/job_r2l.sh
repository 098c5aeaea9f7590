python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for l in exp_libs/libgem_new.so exp_libs/libgem_loc.so; do python scripts/ab_time.py $l --cfg c1; done
timeout 1800 python -m pytest tests -m gpu -x -q -k "c1 or golden or wires or small or cells or activity or noinput" 2>&1 | tail -3
python scripts/prof_run.py --cfg c1 --phases 2>&1 | tail -5
