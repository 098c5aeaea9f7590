rm -rf .cache
( time timeout 1200 python bench.py > gpurun_out/r2x_bench_default.json 2> gpurun_out/r2x_bench_default.err ) 2> gpurun_out/r2x_bench_default.time
tail -c 200 gpurun_out/r2x_bench_default.json; cat gpurun_out/r2x_bench_default.time
bash scripts/gpu_job.sh r2x smoke pytest bench:c1 bench:c2 bench:c4 bench:c5 ref:c3 ncu:c3 ncu:c5 sanitize:memcheck sanitize:racecheck sanitize:synccheck
