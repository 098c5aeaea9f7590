# C3 word-mode mapping variants (partition balance), cycles/s on one box
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_dac_guozwlr25_b200/csrc/libgem.so
for O in "part_size=7000 max_parts=148 levels=10 key=2 merge_ratio=0.6 merge_cap=9000 words=1" \
         "part_size=6500 max_parts=148 levels=10 key=2 merge_ratio=0.6 merge_cap=8500 words=1" \
         "part_size=7000 max_parts=148 levels=10 key=2 merge_ratio=0.6 merge_cap=8000 words=1" \
         "part_size=6000 max_parts=148 levels=10 key=2 merge_ratio=0.6 merge_cap=9000 words=1" \
         "part_size=7000 max_parts=148 levels=10 key=2 merge_ratio=0.5 merge_cap=9000 words=1" ; do
  timeout 400 python scripts/ab_time.py $L --cfg c3 --steps 5 --map-opts "$O" 2>&1 | tail -1
done
