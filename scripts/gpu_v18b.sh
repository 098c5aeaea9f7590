# HEAD: full GPU parity suite (incl. degenerate cases) and the remaining bench lines
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_v18b.log 2>&1; tail -1 gpurun_out/pytest_gpu_v18b.log
for w in c1 c2 c4; do
  timeout 900 python bench.py --workload $w --steps 10 --warmup 3 > gpurun_out/bench_v18_$w.json 2> gpurun_out/bench_v18_$w.err; tail -c 200 gpurun_out/bench_v18_$w.json
done
