mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "" "levels=10" "levels=10 max_warps=1" "levels=10 max_warps=2" "levels=10 max_warps=4"; do
  echo "== $o"; timeout 600 python scripts/prof_run.py --cfg c1 --cycles 1000 --phases --map-opts "$o" 2>&1 | grep "launch 1\|critical CTA [0-9]\|rror" | cut -c1-200
done
