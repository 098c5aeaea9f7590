python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_dac_guozwlr25_b200/csrc/libgem.so
for o in "levels=10 key=2 part_size=2500" "levels=10 key=2 part_size=2000" "levels=10 key=2 part_size=3000" "levels=10 key=2 part_size=2500 km1=0" "levels=10 key=2 part_size=1800 merge_ratio=0.6"; do
python scripts/ab_time.py $L --cfg c2 --map-opts "$o"
done
for o in "stages=1 levels=10 key=2 part_size=16000" "stages=1 levels=10 key=2 part_size=30000" "stages=1 levels=10 key=2 part_size=22000 merge_ratio=0.6 merge_cap=40000"; do
python scripts/ab_time.py $L --cfg c4 --cycles 200 --steps 5 --map-opts "$o"
done
