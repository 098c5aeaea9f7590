export EXP_CFGS="c1 c3"
python scripts/experiment.py "" "-DEXP_NO_TOP" "-DEXP_NO_LOAD" "-DEXP_NO_GATHER" "-DEXP_NO_TOP -DEXP_NO_LOAD -DEXP_NO_GATHER" "-DEXP_NO_FOLD" 2>&1 | grep -v "warning\|\^\|^$\|Remark\|__attribute\|L0 = nullptr\|ldsb"
