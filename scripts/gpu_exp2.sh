export EXP_CFGS="c3"
python scripts/experiment.py "" "-DEXP_SAME_L" "-DEXP_NO_WAIT" "-DEXP_NO_GATHER" "-DEXP_NO_WAIT -DEXP_NO_GATHER" 2>&1
