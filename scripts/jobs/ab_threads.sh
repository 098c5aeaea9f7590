for cfg in c3 c2; do
O=$(python -c "from tests.common import MAP_OPTS; print(MAP_OPTS['$cfg'])")
for L in libgem_256.so libgem_512.so; do for f in 256 512; do
  echo "== $L fill=$f $cfg"; timeout 300 python scripts/ab_time.py $L --cfg $cfg --steps 6 --map-opts "$O word_fill=$f" 2>&1 | tail -1
done; done; done
