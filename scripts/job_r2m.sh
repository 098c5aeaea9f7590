python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_dac_guozwlr25_b200/csrc/libgem.so
B="part_size=8000 max_parts=148 levels=10 merge_ratio=0.6 merge_cap=12000"
python scripts/ab_time.py $L --cfg c3 --map-opts "$B key=2 km1_pins=1024"
python scripts/ab_time.py $L --cfg c3 --map-opts "$B key=0 km1_pins=1024"
python scripts/ab_time.py $L --cfg c3 --map-opts "$B key=0"
python scripts/ab_time.py $L --cfg c5 --streams 4096 --cycles 100 --map-opts "refine=0 lanes=1 key=2 merge_cap=60000 lane_words=7000 levels=10 merge_ratio=0.5 km1_pins=1024"
python scripts/ab_time.py $L --cfg c5 --streams 4096 --cycles 100 --map-opts "refine=0 lanes=1 key=0 merge_cap=60000 lane_words=7000 levels=10 merge_ratio=0.5 km1_pins=1024"
