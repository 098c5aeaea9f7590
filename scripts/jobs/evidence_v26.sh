# v26: C3 mapped for word mode balance (part_size=7000 merge_cap=9000): default bench from a fresh
# cache, C3 GPU tests (word + bit-packed), ncu launch list + capture of the word kernel
rm -rf .cache
( time timeout 1500 python bench.py > gpurun_out/v26_bench_default.json 2> gpurun_out/v26_bench_default.err ) 2> gpurun_out/v26_bench_default.time
tail -c 200 gpurun_out/v26_bench_default.json; cat gpurun_out/v26_bench_default.time
bash scripts/gpu_job.sh v26 pytest:c3 ncu:c3
