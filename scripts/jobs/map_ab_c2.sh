# C2 word-mode mapping variants, cycles/s on one box
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_dac_guozwlr25_b200/csrc/libgem.so
for O in "levels=10 key=2 part_size=2000 words=1" "levels=10 key=2 parts=76 words=1" "levels=10 key=2 parts=110 words=1" \
         "levels=10 key=2 parts=148 words=1" "levels=10 key=2 part_size=1200 max_parts=148 words=1"; do
  timeout 400 python scripts/ab_time.py $L --cfg c2 --steps 5 --map-opts "$O" 2>&1 | tail -1
done
