# final check at HEAD: default bench from a fresh cache + smoke
rm -rf .cache
( time timeout 1500 python bench.py > gpurun_out/v27_bench_default.json 2> gpurun_out/v27_bench_default.err ) 2> gpurun_out/v27_bench_default.time
python -c "import json;d=json.load(open('gpurun_out/v27_bench_default.json'));r=d['roofline'];print(round(d['value']), round(d['e2e']['value']), round(r['frac'],3), d['parity']['po_ok'], d['clocks'])"
cat gpurun_out/v27_bench_default.time | head -2
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
