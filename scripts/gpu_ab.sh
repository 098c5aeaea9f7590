# A/B: every exp_libs/libgem_*.so on one box, C3 (phases) and optional C5; EXP_CFG selects
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
for lib in exp_libs/libgem_*.so; do
  for cfg in ${EXP_CFG:-c3}; do
    if [ $cfg = c5 ]; then extra="--streams 4096 --cycles 100"; else extra="--cycles 1000"; fi
    echo "== $lib $cfg"; GEM_EXP_LIB=$PWD/$lib timeout 600 python scripts/prof_run.py --cfg $cfg $extra --phases 2>&1 | grep "launch 1\|critical CTA\|lane phases\|Error" | cut -c1-260
  done
done
done
