# round-2 evidence v25 (final: balanced word scheduling): default bench from a fresh cache (C3),
# fresh cache (C3), C1/C2/C4/C5 lines, reference arm, ncu launch list + capture of C3 and C5
rm -rf .cache
( time timeout 1500 python bench.py > gpurun_out/v25_bench_default.json 2> gpurun_out/v25_bench_default.err ) 2> gpurun_out/v25_bench_default.time
tail -c 300 gpurun_out/v25_bench_default.json; cat gpurun_out/v25_bench_default.time
bash scripts/gpu_job.sh v25 bench:c1 bench:c2 bench:c4 bench:c5 ref:c3 ncu:c3 ncu:c5
bash scripts/jobs/gpu_tests.sh
