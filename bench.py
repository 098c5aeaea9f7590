"""GEM hot-path benchmark (driver contract).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gem|reference]
                  [--workload c3] [--streams S] [--cycles C]

A "step" = one gem_step over C simulated cycles (default 1000) of the whole
hot path (global read, layers, endpoint commit, RAM, grid barriers) for S
streams per GPU of the workload netlist (default C3: ~1M live ANDs, 32K
flops, 2 RAM blocks; BASELINE.json metric "simulated cycles/sec at 1M AIG
nodes").  value = simulated stream-cycles/s summed over all ranks (weak
scaling: each rank simulates its own streams; N>1 adds the NCCL gather of the
PO traces to rank 0 inside every step).

The L2 (126 MB) is flushed between timed steps by writing a 512 MB buffer
(the C3 program, ~36 MB, would otherwise stay L2-resident across steps).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "simulated cycles/sec at 1M AIG nodes (1 B200); gate-evals/s; batched 1/2/4/8 GPU"
UNIT = "cycles/s"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        d["_source"] = "measured"
        return d
    d = dict(PEAKS_FALLBACK)
    d["_source"] = "fallback"
    return d


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = "index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active," \
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown," \
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def start(self):
        def run():
            while not self._stop.is_set():
                try:
                    out = subprocess.run(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                         timeout=5).stdout.strip()
                    if out:
                        self.rows.append([x.strip() for x in out.split(",")])
                except Exception:
                    pass
                self._stop.wait(0.2)
        self._t = threading.Thread(target=run, daemon=True)
        self._t.start()

    def stop(self) -> dict:
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for k, n in enumerate(names):
                if len(r) > 5 + k and r[5 + k].lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def ncu_traffic(cfg: str, kernel: str, cycles: int):
    """dram read+write bytes of one launch of `kernel` from the newest (highest _vNN) committed
    `--set full` capture summary (profiles/rNN/ncu_<cfg>_*.json, written by
    scripts/ncu_summary.py) taken at the same cycles per launch; else None."""
    import glob
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    best = None
    for f in glob.glob(os.path.join(ROOT, "profiles", "r*", f"ncu_{cfg}_*.json")):
        try:
            d = json.load(open(f))
            if d.get("capture_cycles") != cycles or kernel not in d.get("kernel", kernel):
                continue
            c, u = d["capture"], d["capture_units"]
            t = sum(float(c[k]) * scale[u[k]] for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
            import re
            mv = re.search(r"_v(\d+)\.json$", f)
            m = (int(mv.group(1)) if mv else -1, os.path.getmtime(f))   # newest version tag, then mtime
            if best is None or m > best[0]:
                best = (m, t, os.path.relpath(f, ROOT))
        except Exception:
            continue
    return (best[1], best[2]) if best else (None, None)


def ncu_pipes(cfg: str, kernel: str, cycles: int, n_sms: int, sm_mhz: float):
    """Pipe utilisation of the same committed `--set full` capture as ncu_traffic:
    shared-memory wavefronts per SM clock (peak 1), alu-pipe busy fraction and
    issue IPC of the captured launch; None if no matching summary."""
    import glob
    import re
    best = None
    for f in glob.glob(os.path.join(ROOT, "profiles", "r*", f"ncu_{cfg}_*.json")):
        try:
            d = json.load(open(f))
            if d.get("capture_cycles") != cycles or kernel not in d.get("kernel", kernel):
                continue
            mv = re.search(r"_v(\d+)\.json$", f)
            key = (int(mv.group(1)) if mv else -1, os.path.getmtime(f))
            if best is None or key > best[0]:
                best = (key, d, os.path.relpath(f, ROOT))
        except Exception:
            continue
    if best is None:
        return None
    c = best[1]["capture"]
    dur_s = float(c["gpu__time_duration.sum"]) * {"ms": 1e-3, "us": 1e-6, "usecond": 1e-6, "msecond": 1e-3}.get(
        best[1]["capture_units"].get("gpu__time_duration.sum", "ms"), 1e-3)
    wf = float(c["l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"])
    return {"smem_wavefronts_per_launch": wf,
            "smem_frac": wf / (dur_s * n_sms * sm_mhz * 1e6),
            "smem_peak": "1 wavefront (128 B) per SM clock",
            "alu_pipe_busy_frac": float(c["sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"]) / 100.0,
            "ipc_per_sm": float(c["sm__inst_executed.avg.per_cycle_active"]), "source": best[2]}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def workload_inputs(cfg: str, n_pi: int, cycles: int, streams, step: int):
    """Synthetic stimulus for one step: C3/C5 recipe (PI0 = reset for the first
    4 cycles of step 0 only, other PIs Bern(1/2)), one seed per (stream, step)."""
    from gen.stimulus import splitmix64, stim_random
    out = []
    base = {"c1": 1, "c2": 102, "c3": 103, "c4": 104, "c5": 105}[cfg]
    for s in streams:
        seed = splitmix64((base ^ (int(s) << 24) ^ step) & 0xFFFFFFFFFFFFFFFF) & 0xFFFFFFFF
        if cfg == "c1":
            from gen.stimulus import stim_c1
            w = stim_c1(cycles, seed, reset_cycles=(0, 1) if step == 0 else ())
        else:
            w = stim_random(n_pi, cycles, seed, reset_pi0_cycles=4 if step == 0 else 0)
            if step and cfg != "c2":
                w[:, 0] &= np.uint32(0xFFFFFFFE)
        out.append(w)
    return np.stack(out)


def cpu_baseline_lanes(eaig_path: str, n_pi: int, target_s: float = 12.0) -> dict:
    """C5: the oracle's 64-lane batched mode, one 64-stream group per host thread."""
    from concurrent.futures import ThreadPoolExecutor
    from gen import stimulus_streams
    from oracle import Oracle
    o = Oracle(eaig_path)
    nth = max(1, os.cpu_count() or 1)
    o.lanes_reset(nth)
    probe = 5
    st = stimulus_streams("c5", n_pi, probe, range(64))
    o.lanes_run(0, st, po=True)
    rate = probe / max(o.last_seconds, 1e-9)           # cycles/s of one 64-lane group
    cycles = int(max(probe, min(5000, rate * target_s)))
    stims = [stimulus_streams("c5", n_pi, cycles, range(64 * g, 64 * g + 64)) for g in range(nth)]
    o.lanes_reset(nth)
    t0 = time.perf_counter()
    with ThreadPoolExecutor(nth) as ex:
        list(ex.map(lambda g: o.lanes_run(g, stims[g], po=True), range(nth)))
    dt = time.perf_counter() - t0
    v = 64 * nth * cycles / dt
    return {"value": v, "unit": UNIT, "cores": nth, "kind": "oracle",
            "sample": f"{64 * nth} of the 4096 C5 streams x {cycles} cycles (64-lane uint64 oracle, "
                      f"{nth} threads, one 64-stream group each)",
            "gate_evals_per_s": v * o.n_ands, "host_nproc": os.cpu_count(), "seconds": dt}


def cpu_baseline(eaig_path: str, n_pi: int, cfg: str, target_s: float = 12.0) -> dict:
    """The oracle as it stands, single-threaded, on a bounded sample (host cores)."""
    from gen import stimulus
    from oracle import Oracle
    if cfg == "c5":
        return cpu_baseline_lanes(eaig_path, n_pi, target_s)
    o = Oracle(eaig_path)
    probe = 50
    st = stimulus("c3" if cfg == "c5" else cfg, n_pi, probe)
    o.run(st, po=True)
    rate = probe / max(o.last_seconds, 1e-9)
    cycles = int(max(probe, min(200000, rate * target_s)))
    o.reset()
    st = stimulus("c3" if cfg == "c5" else cfg, n_pi, cycles)
    o.run(st, po=True)
    v = cycles / o.last_seconds
    return {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{cycles} cycles of {cfg} (1 stream), oracle cycle loop only, single thread",
            "gate_evals_per_s": v * o.n_ands, "host_nproc": os.cpu_count(), "seconds": o.last_seconds}


def cpu_baseline_mt(eaig_path: str, n_pi: int, cfg: str, target_s: float = 8.0) -> dict:
    """the oracle's level-parallel variant on all host cores
    (same results as the single-thread loop; tests/test_oracle.py)."""
    from gen import stimulus
    from oracle import Oracle
    nth = max(1, os.cpu_count() or 1)
    o = Oracle(eaig_path)
    probe = 20
    o.run_mt(stimulus(cfg, n_pi, probe), nth)
    rate = probe / max(o.last_seconds, 1e-9)
    cycles = int(max(probe, min(200000, rate * target_s)))
    o.reset()
    o.run_mt(stimulus(cfg, n_pi, cycles), nth)
    v = cycles / o.last_seconds
    return {"value": v, "unit": UNIT, "cores": nth, "kind": "oracle (level-parallel variant)",
            "sample": f"{cycles} cycles of {cfg} (1 stream), oracle cycle loop only, {nth} threads",
            "gate_evals_per_s": v * o.n_ands, "seconds": o.last_seconds}


WORKLOAD_LABEL = {
    "c1": "c1: 32-bit counter + 32-bit ripple-carry adder + 16-bit LFSR (BASELINE config 1)",
    "c2": "c2: synthetic levelised random AIG, 100K nodes, 4K flops, depth 40 (BASELINE config 2)",
    "c3": "c3: synthetic CPU-core-shaped netlist, 1M AIG nodes, 32K flops, 2 RAM blocks (BASELINE config 3)",
    "c4": "c4: synthetic SoC-shaped netlist, 10M AIG nodes, 256K flops, 24 RAM blocks (BASELINE config 4)",
    "c5": "c5: the c3 netlist with 4096 independent stimulus streams (BASELINE config 5)",
}


def run_reference(args):
    """--impl reference: the CPU oracle as the reference arm (this tier has no
    reference implementation).  Under torchrun only rank 0 runs."""
    ws, rank, local = dist_env()
    if rank != 0:
        return 0
    from tests.common import eaig
    from oracle import Oracle
    from gen import stimulus, stimulus_streams
    cfg = args.workload
    path = eaig(cfg)
    o = Oracle(path)
    n_pi = o.n_pi
    C = args.cycles or {"c4": 200, "c5": 100}.get(cfg, 1000)
    budget = 120.0 / max(1, args.steps + args.warmup)        # seconds of oracle work per step
    if cfg == "c5":
        # 64-lane oracle, one 64-stream group per host thread, bounded cycles per step
        from concurrent.futures import ThreadPoolExecutor
        nth = max(1, os.cpu_count() or 1)
        o.lanes_reset(nth)
        probe = 3
        o.lanes_run(0, stimulus_streams("c5", n_pi, probe, range(64)), po=True)
        rate = probe / max(o.last_seconds, 1e-9)
        per_step = int(max(2, min(C, rate * budget)))
        o.lanes_reset(nth)
        tot_c, tot_s = 0, 0.0
        for k in range(args.warmup + args.steps):
            st = [stimulus_streams("c5", n_pi, per_step, range(64 * g, 64 * g + 64), seed=105 + k)
                  for g in range(nth)]
            t0 = time.perf_counter()
            with ThreadPoolExecutor(nth) as ex:
                list(ex.map(lambda g: o.lanes_run(g, st[g], po=True), range(nth)))
            dt = time.perf_counter() - t0
            if k >= args.warmup:
                tot_c += 64 * nth * per_step
                tot_s += dt
        cores, sample = nth, f"{64 * nth} streams x {per_step} cycles per step (64-lane oracle, {nth} threads)"
    else:
        probe = 20
        o.run(stimulus(cfg, n_pi, probe))
        rate = probe / max(o.last_seconds, 1e-9)
        per_step = int(max(5, min(C, rate * budget)))
        o.reset()
        tot_c, tot_s = 0, 0.0
        for k in range(args.warmup + args.steps):
            st = stimulus(cfg, n_pi, per_step, seed=103 + k)
            o.run(st)
            if k >= args.warmup:
                tot_c += per_step
                tot_s += o.last_seconds
        cores, sample = 1, f"{per_step} cycles per step x {args.steps} steps, single thread, 1 stream"
    v = tot_c / tot_s
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * tot_s / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": WORKLOAD_LABEL[cfg]},
            "reference_sample": {"cycles_per_step": per_step, "oracle_and_gates_in_file": o.n_ands},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def _free_port() -> int:
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(args) -> int:
    """`bench.py --gpus N` outside torchrun: launch N ranks (one per GPU) under
    torch.distributed.run on this node; fail loudly if fewer than N GPUs."""
    import torch
    n = torch.cuda.device_count()
    if n < args.gpus:
        print(f"bench.py: --gpus {args.gpus} but only {n} CUDA device(s) visible", file=sys.stderr)
        return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def _flush_fn(flush, enabled):
    def f(k):
        if enabled:
            flush.fill_(k)
    return f


def time_region(one_step, steps, warmup_offset, flush, dev, ws, dist, kernel_ms=None):
    """Barrier + synchronize on both sides; one CUDA-event pair per step on the
    launch stream (recorded inside one_step); clocks sampled during the region;
    kernel_ms() = libgem's own event pair around the step's kernel launch."""
    import torch
    clocks = ClockSampler(dev.index)
    clocks.start()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    evs, kms = [], []
    for k in range(steps):
        flush(k)
        e = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
        one_step(warmup_offset + k, e)
        evs.append(e)
        if kernel_ms is not None:
            kms.append(kernel_ms())
    torch.cuda.synchronize(dev)
    if ws > 1:
        dist.barrier()
    return clocks.stop(), evs, kms


def rejected(c):
    bad = {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}
    low = (c.get("sm_mhz") and c.get("sm_max_mhz") and c["sm_mhz"] < 0.85 * c["sm_max_mhz"]
           and not c.get("reasons"))
    return bool(bad & set(c.get("reasons") or [])) or bool(low)


def max_over_ranks(x, dev, ws, dist):
    import torch
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    if ws > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def parity_check(cfg, path, sim_out, stims, C, state=None):
    """Bench-time parity (SURVEY §8(d) `parity{}`): the GPU's first step (from
    reset) against the oracle on the same inputs.  Single stream: the first
    min(C, budget) cycles of stream 0 (+ final flops when all C are checked);
    batched: the first 64 streams (one 64-lane oracle group), all C cycles."""
    from oracle import Oracle
    o = Oracle(path)
    if stims.shape[0] >= 64 and cfg == "c5":
        o.lanes_reset(1)
        r = o.lanes_run(0, stims[:64], po=True)
        po_ok = bool(np.array_equal(sim_out[:64], r["po"]))
        st_ok = None
        if state is not None:
            st_ok = all(np.array_equal(state[s], o.lanes_get_state(0, s)) for s in range(64))
        return {"po_ok": po_ok, "state_ok": st_ok, "cycles_checked": C, "streams_checked": 64,
                "oracle": "64-lane oracle group, streams 0-63 of rank 0"}
    probe = min(C, 20)
    o.run(stims[0, :probe])
    rate = probe / max(o.last_seconds, 1e-9)
    n = int(min(C, max(probe, rate * 6.0)))
    o.reset()
    r = o.run(stims[0, :n])
    po_ok = bool(np.array_equal(sim_out[0, :n], r["po"]))
    st_ok = bool(np.array_equal(state[0], o.get_state())) if (state is not None and n == C) else None
    return {"po_ok": po_ok, "state_ok": st_ok, "cycles_checked": n, "streams_checked": 1,
            "oracle": "single-stream oracle, stream 0 of rank 0"}


def run_workload(cfg, args, ws, rank, dev, dist, total_streams, scaling, do_e2e=True, split=False):
    """Time `args.steps` gem_step calls of `cfg` (after `args.warmup`), max over ranks.
    split: one stream of one design whose partitions are split over the ws
    ranks (row f4, gem_dist_*: peer stores + cross-device barrier each cycle)."""
    import torch
    from paper_conf_dac_guozwlr25_b200 import gem
    from paper_conf_dac_guozwlr25_b200.dist import gather_traces, shard_streams
    from paper_conf_dac_guozwlr25_b200.isa import blob_info
    from tests.common import blob, eaig, MAP_OPTS

    from paper_conf_dac_guozwlr25_b200.dist import connect_split
    s_start, S = shard_streams(total_streams, ws, rank) if not split else (0, 1)
    dkw = {"dist_world": ws, "dist_rank": rank} if split else {}
    opts = MAP_OPTS[cfg] if (args.map_opts is None or cfg != args.workload) else args.map_opts
    if rank == 0:
        b = blob(cfg, opts)
    if ws > 1:
        dist.barrier()
    if rank != 0:
        b = blob(cfg, opts)
    info = blob_info(b)
    stream = torch.cuda.current_stream(dev)
    sim = gem.Simulator(b, device=dev.index, n_streams=S, cuda_stream=stream.cuda_stream, flags=gem.GEM_F_ASYNC,
                        **dkw)
    C = (args.cycles if cfg == args.workload else 0) or {"c4": 200, "c5": 100}.get(cfg, 1000)
    if split:
        connect_split(sim, C)
    gstreams = list(range(s_start, s_start + S))
    n_steps = args.warmup + args.steps
    host_in = [workload_inputs(cfg, info.n_pi, C, gstreams, k) for k in range(min(n_steps, 4))]
    dev_in = [torch.from_numpy(x.view(np.int32)).to(dev) for x in host_in]
    po_dev = torch.empty((S, C, sim.po_words), dtype=torch.int32, device=dev)
    flush_buf = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)
    flush = _flush_fn(flush_buf, not args.no_flush)
    gather_ev = []

    def one_step(k, ev=None):
        # timed region of a step: input staging (D2D copy + lane transpose), the
        # persistent kernel, the PO unpermute into the output tensor
        if ev is not None:
            ev[0].record(stream)
        sim.set_inputs_device(dev_in[k % len(dev_in)], C)
        sim.step(C)
        sim.read_outputs_device(po_dev, C)
        if ev is not None:
            ev[1].record(stream)
        if ws > 1 and total_streams > ws:
            # batched streams: NCCL gather of the PO traces to rank 0, timed separately
            g = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
            g[0].record(stream)
            gather_traces(po_dev, total_streams)
            g[1].record(stream)
            if ev is not None:
                gather_ev.append(g)

    for k in range(args.warmup):
        one_step(k)
    torch.cuda.synchronize(dev)
    clk, evs, kms = time_region(one_step, args.steps, args.warmup, flush, dev, ws, dist, sim.last_step_ms)
    flag = 1.0 if rejected(clk) else 0.0
    if max_over_ranks(flag, dev, ws, dist) > 0:
        first = clk
        gather_ev.clear()
        clk, evs, kms = time_region(one_step, args.steps, args.warmup, flush, dev, ws, dist, sim.last_step_ms)
        clk = dict(clk, remeasured=True, first_run=first)
    step_ms = [a.elapsed_time(b_) for a, b_ in evs]
    tot_ms = max_over_ranks(sum(step_ms), dev, ws, dist)
    gather_ms = max_over_ranks(sum(a.elapsed_time(b_) for a, b_ in gather_ev), dev, ws, dist) if gather_ev else 0.0
    kern_ms = float(np.mean(kms))
    res = {"cfg": cfg, "info": info, "sim_info": sim.info, "C": C, "S": S, "total_streams": total_streams,
           "tot_ms": tot_ms, "step_ms": step_ms, "gather_ms": gather_ms, "clk": clk, "kern_ms": kern_ms,
           "value": total_streams * C * args.steps / (tot_ms / 1e3),
           "value_with_gather": total_streams * C * args.steps / ((tot_ms + gather_ms) / 1e3),
           "scaling": scaling, "path": eaig(cfg)}
    sim.close()
    if not do_e2e:
        return res
    # ---- e2e through the public C ABI with HOST buffers (pinned), copies inside the timed region
    sim_h = gem.Simulator(b, device=dev.index, n_streams=S, **dkw)
    if split:
        connect_split(sim_h, C)
    host_pinned = [torch.from_numpy(x.view(np.int32)).pin_memory() for x in host_in]
    # first call from reset on step 0's inputs: the parity sample below
    sim_h.set_inputs(host_pinned[0].numpy().view(np.uint32))
    sim_h.step(C)
    first_out = sim_h.read_outputs(C)
    first_state = sim_h.read_state()
    for k in range(1, 3):
        sim_h.set_inputs(host_pinned[k % len(host_pinned)].numpy().view(np.uint32))
        sim_h.step(C)
        sim_h.read_outputs(C)
    if ws > 1:
        dist.barrier()
    # L2 flushed before every step as in the device-timed region (outside the
    # clock: each step is timed from the API call to the return of its D2H read)
    e2e_steps = max(3, args.steps // 2)
    e2e_s = 0.0
    for k in range(e2e_steps):
        flush(k + 1)
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        sim_h.set_inputs(host_pinned[k % len(host_pinned)].numpy().view(np.uint32))
        sim_h.step(C)
        sim_h.read_outputs(C)
        e2e_s += time.perf_counter() - t0
    e2e_s = max_over_ranks(e2e_s, dev, ws, dist)
    res["e2e"] = {"value": total_streams * C * e2e_steps / e2e_s, "unit": UNIT,
                  "h2d_bytes_per_step": int(S * C * sim.pi_words * 4),
                  "d2h_bytes_per_step": int(S * C * sim.po_words * 4),
                  "api": "gem_set_inputs(host) + gem_step + gem_read_outputs(host), synchronous C ABI"}
    sim_h.close()
    if rank == 0:
        res["parity"] = parity_check(cfg, eaig(cfg), first_out, host_in[0], C, first_state)
    return res


def roofline(res, peaks, dev):
    """The binding roofline of the dominant kernel."""
    import torch
    from paper_conf_dac_guozwlr25_b200 import gem
    info, C, S, cfg = res["info"], res["C"], res["S"], res["cfg"]
    sm_mhz = res["clk"].get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0)
    n_sms = torch.cuda.get_device_properties(dev).multi_processor_count
    peak_lop3 = n_sms * 64 * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
    hz_kernel = C / (res["kern_ms"] / 1e3)
    achieved_lop3 = info.n_and / 16.0 * hz_kernel * S   # this rank's kernel (per GPU)
    words = bool(res["sim_info"].get("words"))
    kname = "gem_lane_kernel" if res["sim_info"]["lanes"] else "gem_word_kernel" if words else "gem_step_kernel"
    traffic, traffic_src = ncu_traffic(cfg, kname, C)
    alu = {"bound": "alu", "achieved": achieved_lop3 / 1e12, "peak": peak_lop3 / 1e12, "unit": "TLOP3/s",
           "frac": achieved_lop3 / peak_lop3,
           "algorithmic": "N_and/16 LOP3 per stream-cycle (2 LOP3 per 32 gate evals, P:81)",
           "peak_source": f"{n_sms} SMs x 64 LOP3/clk x sm_max_mhz ({peaks['_source']})"}
    alg_bytes = (2 * info.n_flops + info.n_pi + info.n_po) / 8.0 + 12.0 * info.n_rams
    hbm_peak = float(peaks.get("hbm_gbs", 6650))
    hbm = {"bound": "hbm", "program_bytes_per_cycle_if_streamed": info.program_bytes,
           "frac_if_streamed": info.program_bytes * hz_kernel / (hbm_peak * 1e9),
           "ideal_program_bytes": 4 * info.n_and,
           "frac_if_streamed_vs_ideal_4B_per_and": 4 * info.n_and * hz_kernel / (hbm_peak * 1e9),
           "algorithmic_bytes_per_stream_cycle": alg_bytes,
           "algorithmic_bytes_per_launch": alg_bytes * C * S + info.program_bytes,
           "peak_gbs": hbm_peak}
    roof = dict(alu)
    roof["pipes_ncu"] = ncu_pipes(cfg, kname, C, n_sms, float(peaks.get("sm_max_mhz", 1965.0)))
    roof.update({"traffic": traffic, "traffic_unit": "bytes per launch (dram read+write, ncu --set full)",
                 "traffic_source": traffic_src, "kernel": kname, "kernel_ms_per_step": res["kern_ms"],
                 "us_per_layer_critical": 1e6 / hz_kernel / max(1, info.max_layers), "alu": alu, "hbm": hbm})
    if S == 1:
        lay_clk, bar_clk = gem.bench_floor(dev.index, res["sim_info"]["grid"])
        f_hz = float(sm_mhz) * 1e6
        if words:
            # word mode: the chain is the deepest word program's
            # steps, each at least one minimal step (gem_bench_floor_step)
            step_clk = gem.bench_floor_step(dev.index)
            crit = sum(info.stage_max_word_steps())
            floor_hz = f_hz / (crit * step_clk + info.n_stages * bar_clk)
            lat = {"bound": "latency", "achieved": hz_kernel, "peak": floor_hz, "unit": "cycles/s",
                   "frac": hz_kernel / floor_hz, "mode": "words",
                   "step_clk": step_clk, "barrier_clk": bar_clk, "critical_steps": crit, "stages": info.n_stages,
                   "achieved_clk_per_cycle": f_hz / hz_kernel,
                   "achieved_clk_per_critical_step": f_hz / hz_kernel / max(1, crit),
                   "definition": "peak = sm_clock / (sum over stages of the deepest word program's steps x "
                                 "minimal-step clocks + stages x grid-barrier clocks); minimal step = block barrier "
                                 "+ two operand loads + AND + store per thread (gem_bench_floor_step, measured on "
                                 "this GPU in this run)"}
        else:
            crit = sum(info.stage_max_layers())
            floor_hz = f_hz / (crit * lay_clk + info.n_stages * bar_clk)
            lat = {"bound": "latency", "achieved": hz_kernel, "peak": floor_hz, "unit": "cycles/s",
                   "frac": hz_kernel / floor_hz, "mode": "bits",
                   "layer_clk": lay_clk, "barrier_clk": bar_clk, "critical_layers": crit, "stages": info.n_stages,
                   "achieved_clk_per_cycle": f_hz / hz_kernel,
                   "achieved_clk_per_critical_layer": f_hz / hz_kernel / max(1, crit),
                   "definition": "peak = sm_clock / (sum over stages of the deepest partition's layers x "
                                 "minimal-layer clocks + stages x grid-barrier clocks); minimal layer = one "
                                 "dependent gathered load per thread + 13 fold levels + write-out + block barrier "
                                 "(gem_bench_floor, measured on this GPU in this run)"}
        roof["latency_floor"] = lat
        # does the program stream from HBM every cycle?  The committed ncu
        # capture at the same cycles per launch decides (DRAM bytes per cycle
        # vs program bytes); without one, a program larger than half the L2
        # (126 MB) is assumed to stream
        l2_bytes = 126e6
        if traffic is not None:
            streamed = traffic / C > 0.5 * info.program_bytes
            hbm["dram_bytes_per_cycle_ncu"] = traffic / C
        else:
            streamed = info.program_bytes > 0.5 * l2_bytes
        if words:
            streamed = False   # word programs are copied into shared memory once per launch
        hbm["program_streamed"] = streamed
        hbm_floor = hbm_peak * 1e9 / info.program_bytes if streamed else float("inf")
        hbm["floor_cycles_per_s"] = hbm_floor if hbm_floor != float("inf") else None
        if hz_kernel / hbm_floor > hz_kernel / floor_hz:
            roof.update({"bound": "hbm", "achieved": info.program_bytes * hz_kernel / 1e9,
                         "peak": hbm_peak, "unit": "GB/s", "frac": hz_kernel / hbm_floor,
                         "algorithmic": "program bytes per cycle (the whole program streamed from HBM)",
                         "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peaks['_source']})"})
            roof["binding"] = "hbm (program not L2-resident, streamed every cycle)"
        else:
            roof.update({k: lat[k] for k in ("bound", "achieved", "peak", "unit", "frac")})
            roof.update({"algorithmic": "simulated cycles per second of one stream",
                         "peak_source": "latency floor (gem_bench_floor, measured in this run)"})
            roof["binding"] = "latency"
    elif info.lane_ops:
        # LAN2 lane programs: every AND op moves three 4-byte lane
        # words per 32-stream group through shared memory (two operand loads, one
        # result store); the shared-memory pipe (128 B per SM clock) binds before
        # the LOP3 issue does
        smem_bytes = info.lane_ops * 12.0 / 32.0          # per stream-cycle
        peak_smem = n_sms * 128.0 * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
        ach = smem_bytes * hz_kernel * S
        smem = {"bound": "smem", "achieved": ach / 1e9, "peak": peak_smem / 1e9, "unit": "GB/s",
                "frac": ach / peak_smem,
                "algorithmic": f"{info.lane_ops} AND ops x 3 lane words x 4 B per 32 streams per cycle "
                               f"({smem_bytes:.0f} B per stream-cycle)",
                "peak_source": f"{n_sms} SMs x 128 B/clk x sm_max_mhz ({peaks['_source']})"}
        roof["smem"] = smem
        roof.update({k: smem[k] for k in ("bound", "achieved", "peak", "unit", "frac", "algorithmic", "peak_source")})
        roof["binding"] = "shared-memory traffic of the step ops (ALU fraction alongside)"
    else:
        roof["binding"] = "alu (independent streams: issue of LOP3/LDS per lane word)"
    return roof


def host_info() -> dict:
    """The box's host CPU (oracle timings name their cores)."""
    model = None
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu": model}


def mapping_stats(info) -> dict:
    """SURVEY §8(d) mapping fields of the bench line."""
    return {"n_and": info.n_and, "n_and_mapped": info.n_and_mapped, "n_flops": info.n_flops,
            "n_rams": info.n_rams, "parts": info.n_parts, "stages": info.n_stages,
            "max_layers": info.max_layers, "critical_layers": sum(info.stage_max_layers()),
            "levels": info.max_levels, "total_layers": info.total_layers,
            "replication": round(info.replication, 4), "program_bytes": info.program_bytes,
            "bytes_per_and": round(info.bytes_per_and, 3), "slot_util": round(info.slot_util, 4),
            "levels_per_layer": round(info.max_levels / max(1, info.max_layers), 3),
            "n_and_synth": info.n_and_synth, "levels_in": info.levels_in,
            "leaf_util": round(info.total_leaves / max(1, info.total_layers * 8192), 4),
            "lane_ops": info.lane_ops, "lane_steps": info.lane_steps,
            "word_programs": info.has_words, "word_ops": info.word_ops,
            "critical_word_steps": sum(info.stage_max_word_steps()) if info.has_words else None,
            "word_program_bytes": info.word_program_bytes,
            "levels_per_critical_step": round(info.max_levels / max(1, sum(info.stage_max_word_steps())), 3)
            if info.has_words else None}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gem", choices=["gem", "reference"])
    ap.add_argument("--workload", default="c3", choices=["c1", "c2", "c3", "c4", "c5"])
    ap.add_argument("--streams", type=int, default=0,
                    help="TOTAL stimulus streams over all GPUs (0 = 1 per GPU, or 4096 for c5)")
    ap.add_argument("--cycles", type=int, default=0,
                    help="simulated cycles per step (0 = 1000; 200 for c4; 100 for c5)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-batched", action="store_true", help="skip the batched C5 (4096-stream) companion run")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--map-opts", default=None)
    ap.add_argument("--split", action="store_true",
                    help="N>1: split the single design's partitions over the N GPUs (row f4) instead of replicas")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    args.warmup = max(3, args.warmup)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch(args)

    import torch
    import torch.distributed as dist
    ws, rank, local = dist_env()
    if ws != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}", file=sys.stderr)
        return 2
    one_dev = os.environ.get("GEM_BENCH_ONE_DEVICE") == "1"
    if one_dev:
        local = 0
    if not torch.cuda.is_available() or torch.cuda.device_count() < (local + 1):
        print("bench.py: no CUDA device for this rank (there is no CPU fallback)", file=sys.stderr)
        return 2
    # GEM_BENCH_ONE_DEVICE=1 (tests of the N>1 code paths on a 1-GPU box): every
    # rank on cuda:0, gloo process group (NCCL refuses two ranks on one device)
    if ws > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.cuda.set_device(local)
        if one_dev:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", local if ws > 1 else 0)

    cfg = args.workload
    split = args.split and ws > 1
    if split and (cfg == "c5" or args.streams):
        print("bench.py: --split runs one stream of a single design (c1-c4)", file=sys.stderr)
        return 2
    total = 1 if split else (args.streams or (4096 if cfg == "c5" else ws))
    scaling = "strong" if (args.streams or cfg == "c5" or split) else "weak"
    main_res = run_workload(cfg, args, ws, rank, dev, dist, total, scaling, split=split)
    batched = None
    if cfg != "c5" and not args.no_batched:
        b = run_workload("c5", args, ws, rank, dev, dist, 4096, "strong", do_e2e=False)
        batched = b

    if rank == 0:
        from tests.common import eaig
        peaks = _peaks()
        info = main_res["info"]
        roof = roofline(main_res, peaks, dev)
        cpu = cpu_mt = None
        if ws == 1 and not args.no_cpu_baseline:
            cpu = cpu_baseline(eaig(cfg), info.n_pi, cfg)
            if cfg != "c5":   # C5's baseline already runs one 64-lane group per host core
                cpu_mt = cpu_baseline_mt(eaig(cfg), info.n_pi, cfg)
        sim_info = main_res["sim_info"]
        C, S = main_res["C"], main_res["S"]
        lanes = sim_info["lanes"]
        n_launch = 3 if lanes else 2     # (+ to_lanes_kernel for lane mode)
        cfgd = {"workload": WORKLOAD_LABEL[cfg], "streams_total": total, "streams_per_gpu": S,
                "cycles_per_step": C, "stream_group": sim_info["group"], "grid": sim_info["grid"],
                "mapping": mapping_stats(info),
                "l2": "flushed between timed steps (512 MB write), device-timed and e2e"
                if not args.no_flush else "not flushed",
                "parallelism": (f"one design split over {ws} GPUs: {info.n_parts} partitions by gem_dist_owner, "
                                "peer stores of committed words + cross-device barrier per stage (row f4)"
                                if split else
                                f"streams sharded over {ws} GPU(s), NCCL gather of PO traces"
                                if (ws > 1 and total > ws) else
                                f"{ws} independent replicas (single design: replicas only, DESIGN.md §8)"
                                if ws > 1 else "1 GPU")}
        line = {"metric": METRIC, "value": main_res["value"], "unit": UNIT, "n_gpus": ws, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": main_res["tot_ms"] / args.steps, "higher_is_better": True,
                "scaling": scaling, "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": cfgd,
                "gate_evals_per_s": main_res["value"] * info.n_and,
                "clocks": main_res["clk"], "gpu_launches": args.steps * (n_launch + (1 if lanes else 0)),
                "gpu_launches_detail": ("per step: to_lanes_kernel (input transpose) + gem_lane_kernel (persistent, "
                                        "all cycles) + from_lanes_kernel + unpermute_kernel") if lanes else
                                       ("per step: 1 %s (persistent, all cycles) + 1 unpermute_kernel" %
                                        ("gem_word_kernel" if main_res["sim_info"].get("words") else "gem_step_kernel")),
                "timed_region": "per step: input staging (D2D copy of the step's PI words"
                                + (" + lane transpose" if lanes else "") + "), gem_step, PO unpermute",
                "e2e": main_res.get("e2e"), "roofline": roof, "parity": main_res.get("parity"),
                "host": host_info(), "seeds": {"netlist": {"c1": None, "c2": 2, "c3": 3, "c4": 4, "c5": 3}[cfg],
                                               "stimulus": "splitmix64(base ^ stream << 24 ^ step), base "
                                                           f"{ {'c1': 1, 'c2': 102, 'c3': 103, 'c4': 104, 'c5': 105}[cfg] }"},
                "cpu_baseline": cpu, "cpu_baseline_mt": cpu_mt,
                "step_ms": {"min": min(main_res["step_ms"]), "median": float(np.median(main_res["step_ms"])),
                            "max": max(main_res["step_ms"])}}
        if main_res["gather_ms"]:
            line["nccl_gather_ms_per_step"] = main_res["gather_ms"] / args.steps
            line["value_with_gather"] = main_res["value_with_gather"]
        if batched is not None:
            bi = batched["info"]
            line["batched"] = {
                "workload": WORKLOAD_LABEL["c5"], "metric": "stream-cycles/s (4096 streams, strong scaling)",
                "value": batched["value"], "unit": "stream-cycles/s", "n_gpus": ws,
                "streams_total": 4096, "streams_per_gpu": batched["S"], "cycles_per_step": batched["C"],
                "ms_per_step": batched["tot_ms"] / args.steps,
                "nccl_gather_ms_per_step": batched["gather_ms"] / args.steps if ws > 1 else 0.0,
                "value_with_gather": batched["value_with_gather"],
                "gate_evals_per_s": batched["value"] * bi.n_and,
                "kernel_ms_per_step": batched["kern_ms"], "mapping": mapping_stats(bi),
                "clocks": batched["clk"], "scaling": "strong"}
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
