# why C3's e2e (host buffers) reads ~2% above the device-timed value: the same bench with the
# nvidia-smi clock sampler disabled (monkeypatched, experiment only)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for i in 1 2; do
python - <<'PY' 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('no-sampler', d['value'], d['e2e']['value'], d['roofline']['kernel_ms_per_step'])"
import sys; sys.argv = ["bench.py", "--no-cpu-baseline"]
import bench
bench.ClockSampler.start = lambda self: None
bench.main()
PY
python bench.py --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sampler', d['value'], d['e2e']['value'], d['roofline']['kernel_ms_per_step'])"
done
