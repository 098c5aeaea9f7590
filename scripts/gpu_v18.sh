# end-of-round check at HEAD: build + smoke, GPU parity tests, default bench (C3), C5 and C4 lines, reference arm
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_v18.log 2>&1; tail -1 gpurun_out/smoke_v18.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v18.log 2>&1; tail -1 gpurun_out/pytest_gpu_v18.log
timeout 600 python bench.py > gpurun_out/bench_v18_c3.json 2> gpurun_out/bench_v18_c3.err; tail -c 300 gpurun_out/bench_v18_c3.json
timeout 600 python bench.py --workload c5 --steps 10 --warmup 3 > gpurun_out/bench_v18_c5.json 2> gpurun_out/bench_v18_c5.err; tail -c 300 gpurun_out/bench_v18_c5.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_v18_ref.json 2> gpurun_out/bench_v18_ref.err; tail -c 300 gpurun_out/bench_v18_ref.json
