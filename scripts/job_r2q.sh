rm -rf .cache
( time timeout 1200 python bench.py > gpurun_out/r2q_bench_default.json 2> gpurun_out/r2q_bench_default.err ) 2> gpurun_out/r2q_bench_default.time
tail -c 300 gpurun_out/r2q_bench_default.json; cat gpurun_out/r2q_bench_default.time
timeout 300 python bench.py --gpus 2 > gpurun_out/r2q_gpus2.log 2>&1; echo "gpus2 rc=$?"; tail -2 gpurun_out/r2q_gpus2.log
bash scripts/gpu_job.sh r2q smoke pytest bench:c1 bench:c2 bench:c4 bench:c5 ref:c3 ncu:c3 ncu:c5
