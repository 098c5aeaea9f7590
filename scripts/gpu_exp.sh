EXP_CFGS="c1 c3" python scripts/experiment.py "" "-DGEM_TOP_ATOMIC" 2>&1 | grep -v "warning\|Remark\|^\s*$\|\^\|declared but\|const uint32_t\|__attribute"
