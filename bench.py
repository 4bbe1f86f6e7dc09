#!/usr/bin/env python
"""Benchmark of libipt's 3-stage in-place transposition on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload sweep|c1|c3|c4|c5|table2]

Metric (BASELINE.json): in-place transpose effective GB/s = 2*M*N*elem_bytes / time
(PAPER.md P:56), whole job (all ranks); also reported as a fraction of the measured HBM
peak scaled by the stage count S.

Default workload (N = 1): BASELINE.json configs[1], the float32 shape sweep with
M, N in [1000, 20000].  One step = one in-place transpose of
every matrix of the sweep (each matrix alternates between M x N and N x M from step to
step; every matrix is larger than L2, so no flush is needed between steps).  Multi-GPU:
every rank runs the same per-GPU work on its own GPU (weak scaling, no collective on the
data path); --workload c5 instead shards 512 matrices across ranks (strong scaling).

Reference arm (--impl reference): the repo's CPU oracle (oracle/, plain single-thread C
cycle following), timed on the host on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "in-place transpose effective GB/s (2·M·N·bytes/time), % of B200 HBM peak"

SWEEP = [(7200, 18000), (18000, 7200), (16384, 16384), (12800, 15000), (19200, 10000),
         (9998, 12288), (14803, 8192), (20000, 20000)]
WORKLOADS = {
    "sweep": dict(name="configs[1] shape sweep, float32, M,N in [1000,20000]", shapes=SWEEP, eb=4),
    "c1": dict(name="configs[0] single 1800x7200 float32", shapes=[(1800, 7200)], eb=4),
    "c3": dict(name="configs[2] skinny 1000000x256 float32", shapes=[(1_000_000, 256)], eb=4),
    "c4": dict(name="configs[3] large 20000x30000 float64", shapes=[(20000, 30000)], eb=8),
    "c5": dict(name="configs[4] batch of 512 4096x3000 float32", shapes=[(4096, 3000)], eb=4,
               batch=512),
    # the paper's Table 2 shapes (~12.9 M single-precision elements each; K20:
    # 18.7-20.7 GB/s) -- a secondary line for the paper comparison, not the headline
    "table2": dict(name="paper Table 2 shapes (P:277-282), float32", shapes=[
        (7200, 1800), (5100, 2500), (4000, 3200), (3300, 3900), (2500, 5100), (1800, 7200)], eb=4),
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------------ helpers
def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class NvmlClockSampler:
    """SM clocks / clock-event (throttle) reasons sampled every ~2 ms by NVML in a thread
    during the timed region (nvidia-smi -lms cannot sample a 50 ms region usefully)."""

    NAMES = {"hw_slowdown": "nvmlClocksEventReasonHwSlowdown",
             "hw_thermal_slowdown": "nvmlClocksEventReasonHwThermalSlowdown",
             "sw_thermal_slowdown": "nvmlClocksEventReasonSwThermalSlowdown",
             "sw_power_cap": "nvmlClocksEventReasonSwPowerCap",
             "hw_power_brake_slowdown": "nvmlClocksEventReasonHwPowerBrakeSlowdown"}

    def __init__(self, device: int):
        import threading

        import pynvml as nv
        import torch

        self.nv = nv
        nv.nvmlInit()
        h = None
        try:   # CUDA and NVML orders differ under CUDA_VISIBLE_DEVICES: match by PCI id
            pr = torch.cuda.get_device_properties(device)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            h = nv.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            h = nv.nvmlDeviceGetHandleByIndex(device)
        self.h = h
        self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        self.rows = []
        self.stop_ev = threading.Event()
        self.th = threading.Thread(target=self._run, daemon=True)
        self.th.start()

    def sample(self):
        """One sample (also called from the main thread while it waits for the GPU)."""
        nv = self.nv
        try:
            self.rows.append((nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM),
                              nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)))
        except Exception:
            pass

    def _run(self):
        while not self.stop_ev.is_set():
            self.sample()
            self.stop_ev.wait(0.002)

    def stop(self):
        self.stop_ev.set()
        self.th.join(timeout=5)
        if not self.rows:
            return None
        reasons = sorted(n for n, attr in self.NAMES.items()
                         if any(r & getattr(self.nv, attr, 0) for _, r in self.rows))
        return {"sm_mhz": statistics.median(c for c, _ in self.rows), "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(self.rows), "source": "nvml, 2 ms"}


def clock_sampler(device: int):
    try:
        return NvmlClockSampler(device)
    except Exception:
        return ClockSampler(device)


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region (fallback)."""

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={index}", f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        for line in open(self.f.name):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append((float(parts[1]), float(parts[2]), parts[5:9]))
            except ValueError:
                continue
        os.unlink(self.f.name)
        if not rows:
            return None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for _, _, r in rows for i, v in enumerate(r) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[0] for r in rows),
                "sm_max_mhz": max(r[1] for r in rows), "reasons": reasons, "samples": len(rows)}


def dist_setup():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# ------------------------------------------------------------ CPU oracle (baseline)
def oracle_sample(shapes, eb, budget_s=12.0, max_mats=None):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload."""
    import numpy as np
    from inputs import seeded
    from oracle import oracle

    oracle.build()
    done_bytes, t_total, used = 0, 0.0, []
    for (M, N) in shapes:
        a = seeded.matrix_np(M, N, eb)
        t0 = time.perf_counter()
        oracle.transpose_inplace(a, M, N)
        dt = time.perf_counter() - t0
        # spot-check the oracle's own result against the definition
        rnd = np.random.default_rng(0)
        ks = rnd.integers(0, M * N, 64)
        i, j = ks // N, ks % N
        assert np.array_equal(a[j * M + i], seeded.values_np(ks, eb))
        done_bytes += 2 * M * N * eb
        t_total += dt
        used.append(f"{M}x{N}")
        del a
        if t_total >= budget_s or (max_mats and len(used) >= max_mats):
            break
    return done_bytes, t_total, used


def run_reference(args, world, rank):
    if rank != 0:
        return 0
    wl = WORKLOADS[args.workload]
    shapes = wl["shapes"]
    # one step = the oracle on one matrix of the workload (bounded: the smallest one)
    sample = min(shapes, key=lambda s: s[0] * s[1])
    for _ in range(args.warmup):
        oracle_sample([sample], wl["eb"], budget_s=0)
    tot_b, tot_t = 0, 0.0
    for _ in range(args.steps):
        b, t, _ = oracle_sample([sample], wl["eb"], budget_s=0)
        tot_b += b
        tot_t += t
    value = tot_b / tot_t / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * tot_t / args.steps, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl["name"], "sample": f"{sample[0]}x{sample[1]} per step",
                   "elem_bytes": wl["eb"]},
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": f"one {sample[0]}x{sample[1]} matrix per step, single thread C"},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# -------------------------------------------------------------------------- ours
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="sweep", choices=sorted(WORKLOADS))
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--queues", type=int, default=4)
    ap.add_argument("--e2e-streams", type=int, default=4)
    ap.add_argument("--e2e-api", default="async", choices=["pipeline", "async"],
                    help="e2e through ipt_transpose_host_async per matrix on --e2e-streams streams "
                         "(default: 80 GB/s) or ipt_transpose_host_pipeline, one call per step "
                         "(76 GB/s: one copy engine per direction)")
    ap.add_argument("--autotune", type=int, default=8,
                    help="candidates timed by ipt_plan_autotune per shape (<2: model plan)")
    ap.add_argument("--stage-events", default="last", choices=["all", "last", "none"],
                    help="per-stage CUDA events (roofline per-kernel times): every timed step, "
                         "the last two (default: an event record between every stage costs "
                         "2.7 %% on the sweep, 17 %% on 50 MB matrices), or none")
    ap.add_argument("--graphs", type=int, default=0,
                    help="1: replay each matrix's plan as a captured CUDA graph (ipt_graph_*) on "
                         "the steps without per-stage events")
    ap.add_argument("--algo", default="3stage", choices=["3stage", "4stage"],
                    help="4stage = the paper's Gustavson/Karlsson baseline (comparison only)")
    args = ap.parse_args()
    world, rank, local = dist_setup()

    if args.impl == "reference":
        return run_reference(args, world, rank)

    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_sunggggh14_b200 as ipt
    from paper_conf_ppopp_sunggggh14_b200.partition import shard
    from inputs import seeded

    assert args.warmup >= 3, "timing rules: at least 3 warm-up steps"
    # one process per GPU; IPT_BENCH_BACKEND=gloo lets the multi-rank logic run on a
    # single-GPU box for testing (ranks then share the device)
    backend = os.environ.get("IPT_BENCH_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    red_dev = dev if backend == "nccl" else torch.device("cpu")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    wl = WORKLOADS[args.workload]
    eb = wl["eb"]
    tdt = torch.int32 if eb == 4 else torch.int64
    stream = torch.cuda.current_stream()

    # ---- matrices resident in HBM, filled on the device by the seeded generator
    mats = []   # (tensor, M, N, count, t0)
    if "batch" in wl:
        M, N = wl["shapes"][0]
        tot = wl["batch"]
        lo, hi = shard(tot, world, rank)          # contiguous block of matrices per rank
        t = torch.empty((hi - lo) * M * N, dtype=tdt, device=dev)
        seeded.fill_device_(t, M, N, eb, t0=lo, count=hi - lo)
        mats.append([t, M, N, hi - lo, lo])
    else:
        for (M, N) in wl["shapes"]:
            t = torch.empty(M * N, dtype=tdt, device=dev)
            seeded.fill_device_(t, M, N, eb)
            mats.append([t, M, N, 1, 0])
    torch.cuda.synchronize()
    plans = {}
    for (t, M, N, cnt, _) in mats:
        if args.autotune > 1 and cnt == 1:
            # measured plan choice (host planning, outside the timed region; data restored)
            plans[(M, N)] = ipt.plan_autotune(t, M, N, args.autotune)
            ipt.transpose_(t, M, N, plan_=plans[(M, N)])
            plans[(N, M)] = ipt.plan_autotune(t, N, M, args.autotune)
            ipt.transpose_(t, N, M, plan_=plans[(N, M)])
        elif args.autotune > 1:
            plans[(M, N)] = ipt.plan_autotune_batched(t, cnt, M, N, args.autotune)
            ipt.transpose_batched_(t, cnt, M, N, plan_=plans[(M, N)])
            plans[(N, M)] = ipt.plan_autotune_batched(t, cnt, N, M, args.autotune)
            ipt.transpose_batched_(t, cnt, N, M, plan_=plans[(N, M)])
        else:
            plans[(M, N)] = ipt.plan(M, N, eb, local)
            plans[(N, M)] = ipt.plan(N, M, eb, local)
    torch.cuda.synchronize()
    ws_bytes = max(ipt.workspace_bytes(p, mt[3]) for mt in mats for p in (plans[(mt[1], mt[2])], plans[(mt[2], mt[1])]))
    ws = torch.empty(max(ws_bytes, 256), dtype=torch.uint8, device=dev)
    orient = [False] * len(mats)   # False: currently M x N; True: currently N x M

    graphs = {}

    def one_step(evs=None):
        for i, (t, M, N, cnt, _) in enumerate(mats):
            a, b = (N, M) if orient[i] else (M, N)
            p = plans[(a, b)]
            if args.graphs and evs is None and args.algo == "3stage":
                key = (i, a, b)          # one captured graph per matrix and orientation
                if key not in graphs:
                    graphs[key] = ipt.Graph(t, a, b, p, count=cnt)
                graphs[key].launch()
            elif cnt > 1:
                ipt.transpose_batched_(t, cnt, a, b, plan_=p,
                                       events=evs[i] if evs is not None else None)
            elif args.algo == "4stage":      # the paper's 4-stage baseline
                ipt.transpose_4stage_(t, a, b, p.m, p.n)
            else:
                ipt.transpose_(t, a, b, plan_=p, workspace=ws,
                               events=evs[i] if evs is not None else None)
            orient[i] = not orient[i]

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()

    # per-stage events for every matrix and every step (created by one record each)
    evs = [[[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in mats]
           for _ in range(args.steps)]
    for s in evs:
        for m in s:
            for e in m:
                e.record()
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size
    resident = any(M * N * eb * cnt <= l2_bytes for (_, M, N, cnt, _) in mats)
    # 4x L2 of flush READS per step (int32 sum over 512 MB) for L2-resident matrices: it
    # evicts the previous step's data (written back here, outside the step's events) and
    # leaves L2 full of clean lines -- a write flush would leave dirty lines whose
    # write-back then lands inside the next timed step
    flush = torch.zeros(128 << 20, dtype=torch.int32, device=dev) if resident else None
    clocks = clock_sampler(local)
    launches0 = ipt.kernel_launch_count()
    orient_before = list(orient)
    torch.cuda.nvtx.range_push("timed")       # ncu --nvtx --nvtx-include "timed/"
    def step_events(s):
        """Per-stage events of step s (cudaEventRecord between the stages of every matrix):
        on every step, only the last two (both orientations), or none (--stage-events)."""
        if args.algo != "3stage" or args.stage_events == "none":
            return None
        if args.stage_events == "last" and s < args.steps - 2:   # last two: both orientations
            return None
        return evs[s]

    if flush is None:
        t_start.record()
        for s in range(args.steps):
            one_step(step_events(s))
        t_end.record()
    else:
        # L2-resident workload: overwrite L2 before every step (outside the step's events)
        # so each step starts cold, as a larger-than-L2 input would
        step_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(args.steps)]
        for s in range(args.steps):
            flush_sum = flush.sum()
            step_ev[s][0].record()
            one_step(step_events(s))
            step_ev[s][1].record()
    # wait with the GIL released so the clock sampler thread runs during the whole region
    last = t_end if flush is None else step_ev[-1][1]
    t_poll = 0.0
    while not last.query():
        if hasattr(clocks, "sample") and time.perf_counter() - t_poll > 0.002:
            clocks.sample()      # the GPU is still running the timed steps
            t_poll = time.perf_counter()
        time.sleep(0.0005)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
    launches = ipt.kernel_launch_count() - launches0
    clk = clocks.stop()
    if flush is None:
        elapsed_ms = t_start.elapsed_time(t_end)
    else:
        elapsed_ms = sum(a.elapsed_time(b) for a, b in step_ev)
    flushed = flush is not None
    del flush
    tmax = torch.tensor([elapsed_ms], dtype=torch.float64, device=red_dev)
    if world > 1:
        dist.barrier()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    elapsed_ms = float(tmax.item())

    # ---- throughput
    bytes_per_step_rank = sum(2 * M * N * eb * cnt for (_, M, N, cnt, _) in mats)
    total_units = bytes_per_step_rank * args.steps * (world if "batch" not in wl else 1)
    if "batch" in wl:
        M, N = wl["shapes"][0]
        total_units = 2 * M * N * eb * wl["batch"] * args.steps
    value_gbs = total_units / (elapsed_ms / 1e3) / 1e9
    peak, peak_src = load_peaks()

    # ---- per-stage (per-kernel) live timing -> roofline of the dominant kernel
    kern_t = {"cycle_global": 0.0, "tile_onchip": 0.0, "square_swap": 0.0}
    kern_bytes = {"cycle_global": 0, "tile_onchip": 0, "square_swap": 0}
    kern_n = {"cycle_global": 0, "tile_onchip": 0, "square_swap": 0}
    stage_scaled = None
    per_shape = {}
    ev_steps = 0
    if args.algo == "3stage":
        orient_sim = list(orient_before)
        S_bytes = 0
        for s in range(args.steps):
            timed = step_events(s) is not None
            ev_steps += timed
            for i, (t, M, N, cnt, _) in enumerate(mats):
                a, b = (N, M) if orient_sim[i] else (M, N)
                p = plans[(a, b)]
                ps = per_shape.setdefault(f"{a}x{b}", {"ms": 0.0, "n": 0, "stage_ms": [0.0, 0.0, 0.0]})
                for st in range(3):
                    v = ipt.VARIANTS[p.variant[st]]
                    if v == "identity":
                        continue
                    S_bytes += 2 * a * b * eb * cnt
                    if not timed:
                        continue
                    dt = evs[s][i][st].elapsed_time(evs[s][i][st + 1])
                    kern_t[v] += dt
                    kern_bytes[v] += 2 * a * b * eb * cnt
                    kern_n[v] += 1
                    ps["ms"] += dt
                    ps["stage_ms"][st] += dt
                ps["n"] += timed
                orient_sim[i] = not orient_sim[i]
        per_shape = {k: v for k, v in per_shape.items() if v["n"]}
        for key, ps in per_shape.items():
            a, b = (int(x) for x in key.split("x"))
            cnt = mats[0][3] if "batch" in wl else 1
            ps["eff_gbs"] = round(2 * a * b * eb * cnt * ps["n"] / (ps["ms"] / 1e3) / 1e9, 1)
            ps["stage_gbs"] = [round(2 * a * b * eb * cnt * ps["n"] / (x / 1e3) / 1e9, 1) if x else None
                               for x in ps["stage_ms"]]
            del ps["ms"], ps["stage_ms"]
        stage_scaled = (S_bytes / (elapsed_ms / 1e3) / 1e9) / peak
    dom = max(kern_t, key=lambda k: kern_t[k]) if any(kern_t.values()) else None
    roofline = None
    if dom:
        achieved = kern_bytes[dom] / (kern_t[dom] / 1e3) / 1e9
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            try:
                traffic = json.load(open(tp)).get(args.workload, {}).get(dom)
            except Exception:
                traffic = None
        roofline = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": peak,
                    "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                    "peak_source": peak_src, "launches": kern_n[dom],
                    "avg_launch_ms": round(kern_t[dom] / max(1, kern_n[dom]), 4),
                    "share_of_step": round(kern_t[dom] / (elapsed_ms * ev_steps / args.steps), 4),
                    "stage_events": f"{args.stage_events} ({ev_steps} of {args.steps} timed steps)",
                    "per_kernel_ms": {k: round(v, 3) for k, v in kern_t.items()}}

    # ---- verification of the final state (sampled, definition-based on device)
    ok = True
    for i, (t, M, N, cnt, t0) in enumerate(mats):
        transposed = orient[i]
        a, b = (M, N) if not transposed else (N, M)   # current shape a x b
        n = M * N
        g = torch.Generator(device="cpu").manual_seed(i)
        for k in range(min(cnt, 3)):
            pos = torch.randint(0, n, (4096,), generator=g).to(dev)
            seg = t[k * n:(k + 1) * n] if cnt > 1 else t
            if transposed:   # position p = j*M + i holds v(i*N + j)
                src = (pos % M) * N + pos // M
            else:
                src = pos
            exp = seeded.values_torch_sample(src + (t0 + k) * n, eb)
            if not torch.equal(seg[pos], exp.to(seg.dtype)):
                ok = False
    del ws
    # ---- e2e through the public host API (H2D + 3 stages + D2H, Sec. 6)
    e2e = None
    if not args.no_e2e and "batch" not in wl:
        hosts = []
        for (_, M, N, _, _) in mats:
            hosts.append([torch.empty(M * N, dtype=tdt, pin_memory=True), M, N])
        for (h, M, N) in hosts:
            tmp = torch.empty(M * N, dtype=tdt, device=dev)
            seeded.fill_device_(tmp, M, N, eb)
            h.copy_(tmp)
            del tmp
        for t_ in mats:
            t_[0] = None
        mats.clear()
        torch.cuda.empty_cache()
        horient = [False] * len(hosts)

        # Several streams (each with its own device staging buffer): the H2D of one matrix
        # overlaps the stages and D2H of the previous one (both PCIe directions busy).
        e2e_streams = [torch.cuda.Stream(device=dev) for _ in range(args.e2e_streams)]

        def e2e_step():
            if args.e2e_api == "pipeline":   # one call: H2D / stages / D2H pipelined across matrices
                shapes = []
                for i, (h, M, N) in enumerate(hosts):
                    shapes.append((N, M) if horient[i] else (M, N))
                    horient[i] = not horient[i]
                ipt.transpose_host_pipeline_([h for (h, _, _) in hosts], shapes)
                return
            cur = torch.cuda.current_stream()
            for st_ in e2e_streams:
                st_.wait_stream(cur)
            for i, (h, M, N) in enumerate(hosts):
                a, b = (N, M) if horient[i] else (M, N)
                ipt.transpose_host_async_(h, a, b, queues=args.queues,
                                          stream=e2e_streams[i % len(e2e_streams)])
                horient[i] = not horient[i]
            for st_ in e2e_streams:
                cur.wait_stream(st_)

        e2e_step()   # warm-up (allocates the device staging buffer)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        w0 = time.perf_counter()
        e0.record()
        for _ in range(args.e2e_steps):
            e2e_step()
        e1.record()
        torch.cuda.synchronize()
        wall = time.perf_counter() - w0
        ems = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(ems, op=dist.ReduceOp.MAX)
        hb = sum(M * N * eb for (_, M, N) in hosts)
        e2e = {"value": round(hb * 2 * args.e2e_steps * world / (float(ems.item()) / 1e3) / 1e9, 3),
               "unit": "GB/s", "h2d_bytes_per_step": hb, "d2h_bytes_per_step": hb,
               "steps": args.e2e_steps, "queues": args.queues, "wall_s": round(wall, 3),
               "api": ("ipt_transpose_host_pipeline (one call per step: H2D of matrix i+1 and D2H of "
                       "matrix i-1 overlap the stages of matrix i; pinned host buffers)"
                       if args.e2e_api == "pipeline" else
                       f"ipt_transpose_host_async on {len(e2e_streams)} streams (pinned host buffers, Sec. 6 queues)")}
        # verify one host result
        (h, M, N) = hosts[0]
        idx = torch.randint(0, M * N, (2048,))
        src = (idx % M) * N + idx // M if horient[0] else idx
        if not torch.equal(h[idx], seeded.values_torch_sample(src, eb).to(h.dtype)):
            ok = False

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        shapes = [(M, N) for (M, N) in wl["shapes"]]
        b, t, used = oracle_sample(shapes, eb, budget_s=12.0)
        cpu = {"value": round(b / t / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"{'+'.join(used)} ({eb}-byte elements), single-thread C cycle following",
               "host_cpus": os.cpu_count()}

    if rank == 0:
        plans_cfg = {f"{M}x{N}": {"m": p.m, "n": p.n, "S": p.n_stages,
                                  "variant": [ipt.VARIANTS[v] for v in p.variant]}
                     for (M, N), p in plans.items()}
        line = {
            "metric": METRIC, "value": round(value_gbs, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(elapsed_ms / args.steps, 4), "higher_is_better": True,
            "scaling": "weak" if "batch" not in wl else "strong", "vs_baseline": None,
            "dtype": "u32" if eb == 4 else "u64", "data": "synthetic",
            "config": {"workload": wl["name"],
                       "shapes": [f"{M}x{N}" for (M, N) in wl["shapes"]],
                       "elem_bytes": eb, "batch": wl.get("batch", 1),
                       "plans": plans_cfg,
                       "l2": ("no flush: every matrix exceeds the 126 MB L2" if not flushed else
                              "L2 flushed before every step (512 MB read, clean lines, outside the step's events; "
                              "time = sum of per-step device times)"),
                       "parallelism": f"replicas x{world}" if "batch" not in wl else f"batch shards x{world}",
                       "algo": args.algo,
                       "planning": (f"ipt_plan_autotune, {args.autotune} candidates per shape "
                                    "(before the timed region)") if args.autotune > 1 else "cost model"},
            "hbm_frac_stage_scaled": round(stage_scaled, 4) if stage_scaled else None,
            "per_shape": per_shape, "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": clk, "verified": ok,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
