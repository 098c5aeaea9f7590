python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python scripts/experiment.py "" "-DEXP_NO_GATHER" "-DEXP_NO_FOLD" "-DEXP_NO_LOAD" "-DEXP_NO_TOP" "-DEXP_NO_GATHER -DEXP_NO_FOLD -DEXP_NO_LOAD -DEXP_NO_TOP"
