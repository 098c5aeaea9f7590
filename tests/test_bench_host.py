"""Host logic of bench.py (no GPU): clock/throttle parsing, the committed ncu
summaries it reads `traffic` from, and the seeded per-step stimulus recipe
(DESIGN.md §4, §9)."""
import numpy as np

import bench


def _sampler(rows):
    s = bench.ClockSampler(0)
    s.rows = rows
    return s.stop()


def test_clock_sampler_reasons_and_median():
    ok = ["0", "1965", "1965", "800.1", "0x0", "Not Active", "Not Active", "Not Active", "Not Active"]
    slow = ["0", "1200", "1965", "990.0", "0x4", "Not Active", "Not Active", "Active", "Active"]
    r = _sampler([ok, ok, slow])
    assert r["sm_mhz"] == 1965.0 and r["sm_max_mhz"] == 1965.0 and r["samples"] == 3
    assert r["reasons"] == ["sw_power_cap", "sw_thermal_slowdown"]
    assert _sampler([ok])["reasons"] == []
    assert _sampler([])["reasons"] == ["unsampled"]


def test_ncu_traffic_matches_capture_cycles():
    # bench.py's launch configurations: C3 1000 cycles, C4 200, C5 100 per gem_step
    for cfg, kern, cyc in [("c3", "gem_step_kernel", 1000), ("c4", "gem_step_kernel", 200),
                           ("c5", "gem_lane_kernel", 100)]:
        t, src = bench.ncu_traffic(cfg, kern, cyc)
        assert t is not None and t > 0 and src.startswith("profiles/"), cfg
        p = bench.ncu_pipes(cfg, kern, cyc, 148, 1965.0)
        assert p is not None and 0 < p["smem_frac"] <= 1 and 0 < p["alu_pipe_busy_frac"] <= 1
    assert bench.ncu_traffic("c3", "gem_step_kernel", 7) == (None, None)


def test_workload_inputs_seeded_per_stream_and_step():
    a = bench.workload_inputs("c5", 70, 16, [0, 1, 2], 0)
    b = bench.workload_inputs("c5", 70, 16, [1], 0)
    c = bench.workload_inputs("c5", 70, 16, [1], 1)
    assert a.shape == (3, 16, 3) and a.dtype == np.uint32
    assert np.array_equal(a[1], b[0])              # a stream's input does not depend on its rank's shard
    assert not np.array_equal(b, c)                # nor repeat across steps
    assert (a[:, :4, 0] & 1).all()                 # reset asserted for the first 4 cycles of step 0
    assert not (c[:, :, 0] & 1).any()              # and released afterwards
    assert not (a[:, :, 2] >> 6).any()             # bits above n_pi stay zero


def test_gpus_flag_launches_ranks_or_fails_loudly():
    """`bench.py --gpus N` outside torchrun relaunches itself with N ranks; with
    fewer than N visible GPUs it exits non-zero with a message (never a silent
    1-GPU run reporting n_gpus = 1)."""
    import os
    import subprocess
    import sys
    import torch
    if torch.cuda.device_count() >= 2:
        import pytest
        pytest.skip("needs a host with fewer than 2 GPUs")
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, bench.__file__, "--gpus", "2"], capture_output=True, text=True, env=env,
                       timeout=300)
    assert r.returncode == 2, (r.returncode, r.stderr[-500:])
    assert "--gpus 2" in r.stderr and "CUDA device" in r.stderr
