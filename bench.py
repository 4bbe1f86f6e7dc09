#!/usr/bin/env python
"""Benchmark of libipt's in-place transposition on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload c5|sweep|c1|c3|c4|table2|primes] [--sub all|none|c1,c4,...]

Metric (BASELINE.json): in-place transpose effective GB/s = 2*M*N*elem_bytes / time
(PAPER.md P:56), whole job (all ranks); also reported as a fraction of the measured HBM
peak scaled by the number S of non-identity stages executed.

Headline (N = 1 and every N): the largest single-GPU BASELINE config, configs[4] = C5, a
batch of 512 independent 4096 x 3000 float32 matrices (25.17 GB), partitioned across the
N ranks by partition.BatchShard (contiguous blocks, no collective on the data path,
P:240).  One step = one ipt_transpose_batched call per rank over its shard: every
matrix, 4096 x 3000, becomes its 3000 x 4096 transpose; the next step reads the same
storage as the next 4096 x 3000 matrices (`--orientation fixed`, default: the configured
shape every step; `alternate` transposes back and forth, 4096 x 3000 and 3000 x 4096 on
alternate steps).  Two extra untimed steps of the reverse shape are reported for context
(`per_shape_reverse`).  The final state is checked on samples against the composition of
every transposition applied since the fill.  Inputs exceed the 126 MB L2: no flush.

Sub-records (N = 1, rank 0, after the headline's timed region; `--sub`): every other
BASELINE config, each matrix timed on its own with per-step CUDA events -- C1 (cold L2),
C3, C4, the paper's Table 2 shapes, the full C2 shape sweep (squares and rectangles
reported separately), and the prime shapes (correctness only).

`--gpus N` without a torchrun environment re-launches this script under
`torch.distributed.run` with N ranks (one process per GPU, 127.0.0.1 rendezvous).

Reference arm (--impl reference): the repo's CPU oracle (oracle/, plain C cycle following,
as it stands) on the host cores: one C5 matrix per core per step.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from inputs import workloads as W  # noqa: E402  (shapes only)

METRIC = "in-place transpose effective GB/s (2·M·N·bytes/time), % of B200 HBM peak"

WORKLOADS = {
    "c5": dict(name="configs[4] batch of 512 independent 4096x3000 float32 matrices",
               shapes=[W.C5_SHAPE], eb=4, batch=W.C5_COUNT),
    "sweep": dict(name="configs[1] shape sweep, float32, M,N in [1000,20000] (SURVEY C2 list)",
                  shapes=W.SWEEP_ALL, eb=4),
    "c1": dict(name="configs[0] single 1800x7200 float32", shapes=W.C1, eb=4),
    "c3": dict(name="configs[2] skinny 1000000x256 float32", shapes=W.C3, eb=4),
    "c4": dict(name="configs[3] large 20000x30000 float64", shapes=W.C4, eb=8),
    "table2": dict(name="paper Table 2 shapes (P:277-282), float32", shapes=W.TABLE2, eb=4),
    "primes": dict(name="prime dimensions (P:319), float32, correctness only", shapes=W.PRIMES, eb=4),
}
SUB_ORDER = ["c1", "c3", "c4", "table2", "sweep", "primes"]


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


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


class NvmlClockSampler:
    """SM clocks / clock-event (throttle) reasons sampled every ~2 ms by NVML in a thread
    during the timed region."""

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


class SmiClockSampler:
    """nvidia-smi clocks / throttle reasons during the timed region (fallback)."""

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


def clock_sampler(device: int):
    try:
        return NvmlClockSampler(device)
    except Exception:
        return SmiClockSampler(device)


def free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


# ------------------------------------------------------------ CPU oracle (baseline)
def oracle_per_core(M, N, eb, t0, cores, rounds=1):
    """The oracle (as it stands, single-threaded C) on `cores` matrices at once, one per
    host thread (ctypes releases the GIL during the C call): C5's embarrassingly parallel
    CPU baseline (BASELINE.md "CPU baseline plan").  Returns (bytes, seconds, cpu_seconds)."""
    from concurrent.futures import ThreadPoolExecutor

    import numpy as np
    from inputs import seeded
    from oracle import oracle

    oracle.build()
    mats = [seeded.matrix_np(M, N, eb, t=t0 + i) for i in range(cores)]
    per = [0.0] * cores

    def one(i):
        a0 = time.perf_counter()
        oracle.transpose_inplace(mats[i], M, N)
        per[i] += time.perf_counter() - a0

    tot = 0.0
    with ThreadPoolExecutor(max_workers=cores) as ex:
        for r in range(rounds):
            w0 = time.perf_counter()
            list(ex.map(one, range(cores)))
            tot += time.perf_counter() - w0
    # spot-check every result against the definition (odd number of rounds = transposed)
    rnd = np.random.default_rng(0)
    for i, a in enumerate(mats):
        ks = rnd.integers(0, M * N, 64)
        if rounds % 2:
            r_, c_ = ks // N, ks % N
            assert np.array_equal(a[c_ * M + r_], seeded.values_np(ks + (t0 + i) * M * N, eb))
    return 2 * M * N * eb * cores * rounds, tot, sum(per)


def oracle_single(M, N, eb):
    """One matrix, one thread: (bytes, seconds)."""
    from inputs import seeded
    from oracle import oracle

    oracle.build()
    a = seeded.matrix_np(M, N, eb)
    t0 = time.perf_counter()
    oracle.transpose_inplace(a, M, N)
    return 2 * M * N * eb, time.perf_counter() - t0


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def run_reference(args, world, rank):
    """--impl reference: the oracle on the host cores, on a bounded sample of the headline
    workload per step (one C5 matrix per core, each step transposes `cores` matrices)."""
    if rank != 0:
        return 0
    wl = WORKLOADS[args.workload]
    M, N = wl["shapes"][0]
    eb = wl["eb"]
    cores = min(host_cores(), 64)
    for _ in range(args.warmup):
        oracle_per_core(M, N, eb, 0, cores) if "batch" in wl else oracle_single(M, N, eb)
    tb, tt = 0, 0.0
    for s in range(args.steps):
        if "batch" in wl:
            b, t, _ = oracle_per_core(M, N, eb, (s * cores) % wl["batch"], cores)
        else:
            b, t = oracle_single(M, N, eb)
        tb += b
        tt += t
    value = tb / tt / 1e9
    sample = (f"{cores} of the {wl.get('batch', 1)} {M}x{N} matrices per step, one per host thread"
              if "batch" in wl else f"one {M}x{N} matrix per step, one thread")
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * tt / args.steps, 3), "higher_is_better": True,
        "scaling": "strong" if "batch" in wl else "weak", "vs_baseline": None,
        "dtype": "u32" if eb == 4 else "u64", "data": "synthetic",
        "config": {"workload": wl["name"], "sample": sample, "elem_bytes": eb},
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": sample, "cpu_model": cpu_model(), "host_cpus": os.cpu_count()},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    emit(line, args)
    return 0


def emit(line, args):
    """Print the bench line; with --record, append it to a JSONL run record as well."""
    print(json.dumps(line), flush=True)
    if getattr(args, "record", None):
        rev = subprocess.run(["git", "rev-parse", "--short", "HEAD"], capture_output=True, text=True,
                             cwd=os.path.dirname(os.path.abspath(__file__))).stdout.strip()
        rec = dict(line, recorded_utc=time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()),
                   git_rev=rev or None, argv=sys.argv[1:])
        with open(args.record, "a") as f:
            f.write(json.dumps(rec) + "\n")


# ---------------------------------------------------------------------- ours: common
def _verify(t, M, N, eb, transposed, t0=0, count=1, nsamp=4096, seed=0, seq=None):
    """Sampled definition check of `count` packed matrices (generator index t0 + k).
    One a x b transpose moves position p = i*b + j to j*a + i; `seq` lists the (a, b)
    transposes applied since the fill, in order (default: one M x N transpose if
    `transposed`, none otherwise), and a sampled position's source is found by undoing
    them in reverse order."""
    import torch
    from inputs import seeded

    n = M * N
    if seq is None:
        seq = [(M, N)] if transposed else []
    g = torch.Generator(device="cpu").manual_seed(seed)
    ok = True
    for k in sorted({0, count // 2, count - 1}):
        pos = torch.randint(0, n, (nsamp,), generator=g).to(t.device)
        seg = t[k * n:(k + 1) * n]
        src = pos.clone()
        for (a, b) in reversed(seq):   # position d = j*a + i came from i*b + j
            src = (src % a) * b + src // a
        exp = seeded.values_torch_sample(src + (t0 + k) * n, eb)
        ok &= bool(torch.equal(seg[pos], exp.to(seg.dtype)))
    return ok


def _stage_rec(ipt, p, cnt, t, a, b, eb, ms):
    """Per-stage record: kernel names and GB/s of the stages that ran."""
    kn = ipt.stage_kernels(p, cnt, t)
    out = []
    for st in range(3):
        if ipt.VARIANTS[p.variant[st]] == "identity":
            continue
        out.append({"stage": st + 1, "kernel": kn[st], "ms": round(ms[st], 4),
                    "gbs": round(2 * a * b * eb * cnt / (ms[st] / 1e3) / 1e9, 1) if ms[st] else None})
    return out


def measure_matrix(ipt, torch, dev, M, N, eb, steps, warmup, autotune, l2_bytes, flush, graphs=False):
    """One matrix on its own: plans (measured), warm-up, `steps` transposes timed one by one
    with CUDA events (orientation alternating; cold L2 for L2-resident matrices), then two
    steps with per-stage events (both orientations), then a sampled definition check."""
    from inputs import seeded

    tdt = torch.int32 if eb == 4 else torch.int64
    t = torch.empty(M * N, dtype=tdt, device=dev)
    seeded.fill_device_(t, M, N, eb)
    torch.cuda.synchronize()
    plans = {}
    for (a, b) in ((M, N), (N, M)):
        if autotune > 1:
            plans[(a, b)] = ipt.plan_autotune(t, a, b, autotune)
        else:
            plans[(a, b)] = ipt.plan(a, b, eb, dev.index)
        ipt.transpose_(t, a, b, plan_=plans[(a, b)])   # leaves the data in (M, N) order again
    resident = M * N * eb <= l2_bytes
    orient = False
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(steps)]

    def one(evs=None):
        nonlocal orient
        a, b = (N, M) if orient else (M, N)
        ipt.transpose_(t, a, b, plan_=plans[(a, b)], events=evs)
        orient = not orient

    for _ in range(warmup):
        one()
    torch.cuda.synchronize()
    for s in range(steps):
        if resident:
            flush.sum()
        ev[s][0].record()
        one()
        ev[s][1].record()
    torch.cuda.synchronize()
    times = [a.elapsed_time(b) for a, b in ev]
    # per-stage events on two extra steps (not in the value)
    stages = {}
    for _ in range(2):
        a, b = (N, M) if orient else (M, N)
        if resident:
            flush.sum()
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        one(evs)
        torch.cuda.synchronize()
        ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(3)]
        stages[f"{a}x{b}"] = _stage_rec(ipt, plans[(a, b)], 1, t, a, b, eb, ms)
    # the same steps replayed as captured CUDA graphs (ipt_graph_create / ipt_graph_launch:
    # no host-side planning or launch API calls per transposition)
    graph_ms = None
    if graphs:
        gr = {(a, b): ipt.Graph(t, a, b, plans[(a, b)]) for (a, b) in ((M, N), (N, M))}
        gtot = 0.0
        for s in range(steps):
            a, b = (N, M) if orient else (M, N)
            if resident:
                flush.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            gr[(a, b)].launch()
            e1.record()
            torch.cuda.synchronize()
            gtot += e0.elapsed_time(e1)
            orient = not orient
        graph_ms = gtot
        del gr
    ok = _verify(t, M, N, eb, orient)
    del t
    torch.cuda.empty_cache()
    tot = sum(times)
    rec = {
        "eff_gbs": round(2 * M * N * eb * steps / (tot / 1e3) / 1e9, 1),
        "ms": round(tot / steps, 4),
        "S": {f"{a}x{b}": p.n_stages for (a, b), p in plans.items()},
        "plan": {f"{a}x{b}": {"m": p.m, "n": p.n} for (a, b), p in plans.items()},
        "stages": stages, "verified": ok,
    }
    sbytes = sum(2 * M * N * eb * plans[(N, M) if (s % 2) else (M, N)].n_stages for s in range(steps))
    rec["hbm_frac_stage_scaled"] = round(sbytes / (tot / 1e3) / 1e9 / load_peaks()[0], 4)
    if graph_ms:
        rec["graph_eff_gbs"] = round(2 * M * N * eb * steps / (graph_ms / 1e3) / 1e9, 1)
    return rec, tot, 2 * M * N * eb * steps


def run_sub(ipt, torch, dev, name, steps, warmup, autotune):
    """Sub-record of one BASELINE config (N = 1): every matrix timed on its own."""
    wl = WORKLOADS[name]
    eb = wl["eb"]
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = torch.zeros(128 << 20, dtype=torch.int32, device=dev)   # 512 MB read flush
    per, agg = {}, {"all": [0.0, 0], "squares": [0.0, 0], "rectangles": [0.0, 0]}
    ok = True
    t0 = time.perf_counter()
    graphs = name in ("c1", "table2")   # single L2-sized matrices: also timed as CUDA graphs
    gagg = [0.0, 0]
    for (M, N) in wl["shapes"]:
        rec, ms, by = measure_matrix(ipt, torch, dev, M, N, eb, steps, warmup, autotune, l2, flush, graphs)
        if "graph_eff_gbs" in rec:
            gagg[0] += by / (rec["graph_eff_gbs"] * 1e9) * 1e3
            gagg[1] += by
        per[f"{M}x{N}"] = rec
        ok &= rec["verified"]
        for k in ("all", "squares" if M == N else "rectangles"):
            agg[k][0] += ms
            agg[k][1] += by
    del flush
    torch.cuda.empty_cache()
    out = {"workload": wl["name"], "elem_bytes": eb, "steps_per_matrix": steps,
           "value": round(agg["all"][1] / (agg["all"][0] / 1e3) / 1e9, 1), "unit": "GB/s",
           "l2": "matrices <= L2 size: 512 MB read flush before every timed step (outside the events)",
           "verified": ok, "wall_s": round(time.perf_counter() - t0, 1)}
    if name == "sweep":
        for k in ("squares", "rectangles"):
            if agg[k][1]:
                out[k] = round(agg[k][1] / (agg[k][0] / 1e3) / 1e9, 1)
    if gagg[1]:
        out["graph_value"] = round(gagg[1] / (gagg[0] / 1e3) / 1e9, 1)
        out["graph_note"] = "the same steps replayed as captured CUDA graphs (ipt_graph_launch)"
    if name == "primes":
        out["note"] = "correctness-only class (P:319: prime dimensions degrade; SURVEY C14)"
    out["per_shape"] = per
    return out


# ------------------------------------------------------------------ ours: headline
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c5", choices=sorted(WORKLOADS))
    ap.add_argument("--sub", default="all",
                    help="sub-records at N = 1: all | none | comma list of " + ",".join(SUB_ORDER))
    ap.add_argument("--sub-steps", type=int, default=6)
    ap.add_argument("--autotune", type=int, default=8,
                    help="candidates timed by ipt_plan_autotune per shape (<2: model plan)")
    ap.add_argument("--e2e-count", type=int, default=64,
                    help="matrices per rank in the e2e timed step (C5 headline)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--orientation", default="fixed", choices=["fixed", "alternate"],
                    help="headline steps: the configured M x N every step (fixed) or M x N and "
                         "N x M on alternate steps")
    ap.add_argument("--record", default=os.environ.get("IPT_BENCH_RECORD"),
                    help="also append the JSON line, with a UTC timestamp and the git revision, "
                         "to this JSONL run-record file")
    args = ap.parse_args()

    # --gpus N outside torchrun: re-launch under torch.distributed.run, one rank per GPU
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
               f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1",
               f"--master-port={free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        log("[bench] spawning", " ".join(cmd))
        return subprocess.call(cmd)

    from paper_conf_ppopp_sunggggh14_b200 import partition as part

    world, rank, local = part.dist_env()
    if world != args.gpus:
        log(f"[bench] WORLD_SIZE={world} but --gpus {args.gpus}")
        return 2
    if args.impl == "reference":
        return run_reference(args, world, rank)

    import torch

    import paper_conf_ppopp_sunggggh14_b200 as ipt
    from inputs import seeded

    assert args.warmup >= 3, "timing rules: at least 3 warm-up steps"
    # one process per GPU; IPT_BENCH_BACKEND=gloo runs the multi-rank logic on one GPU
    backend = os.environ.get("IPT_BENCH_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    red_dev = dev if backend == "nccl" else torch.device("cpu")
    world, rank = part.init_ranks(backend, dev)
    wl = WORKLOADS[args.workload]
    eb = wl["eb"]
    tdt = torch.int32 if eb == 4 else torch.int64

    # ---- the headline workload resident in HBM, filled on the device by the generator
    if "batch" in wl:
        M, N = wl["shapes"][0]
        sh = part.BatchShard(wl["batch"], M, N, eb, world, rank)
    else:   # a list of single matrices: every rank transposes all of them (replicas)
        sh = None
    mats = []   # [tensor, M, N, count, t0]
    if sh is not None:
        t = torch.empty(max(1, sh.count) * M * N, dtype=tdt, device=dev)
        if sh.count:
            seeded.fill_device_(t, M, N, eb, t0=sh.lo, count=sh.count)
        mats.append([t, M, N, sh.count, sh.lo])
    else:
        for (M, N) in wl["shapes"]:
            t = torch.empty(M * N, dtype=tdt, device=dev)
            seeded.fill_device_(t, M, N, eb)
            mats.append([t, M, N, 1, 0])
    torch.cuda.synchronize()
    plans = {}
    for (t, M, N, cnt, _) in mats:
        if cnt == 0:
            continue
        for (a, b) in ((M, N), (N, M)):
            if args.autotune > 1 and cnt > 1:
                plans[(a, b)] = ipt.plan_autotune_batched(t, cnt, a, b, args.autotune)
            elif args.autotune > 1:
                plans[(a, b)] = ipt.plan_autotune(t, a, b, args.autotune)
            else:
                plans[(a, b)] = ipt.plan(a, b, eb, local)
            ipt.transpose_batched_(t, cnt, a, b, plan_=plans[(a, b)])   # back to M x N
    torch.cuda.synchronize()
    orient = [False] * len(mats)
    seqs = [[] for _ in mats]   # transposes applied since the fill (the setup above is net identity)
    fixed = args.orientation == "fixed"

    def one_step(evs=None, reverse=False):
        for i, (t, M, N, cnt, _) in enumerate(mats):
            if cnt == 0:
                continue
            if fixed:
                a, b = (N, M) if reverse else (M, N)
            else:
                a, b = (N, M) if orient[i] else (M, N)
                orient[i] = not orient[i]
            ipt.transpose_batched_(t, cnt, a, b, plan_=plans[(a, b)],
                                   events=evs[i] if evs is not None else None)
            seqs[i].append((a, b))

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()

    # per-stage events on the last two timed steps, created up front
    n_ev = 2
    evs = [[[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in mats]
           for _ in range(n_ev)]
    for s in evs:
        for m in s:
            for e in m:
                e.record()
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size
    resident = any(0 < M * N * eb * cnt <= l2_bytes for (_, M, N, cnt, _) in mats)
    flush = torch.zeros(128 << 20, dtype=torch.int32, device=dev) if resident else None
    torch.cuda.synchronize()
    part.barrier()
    torch.cuda.synchronize()
    clocks = clock_sampler(local)
    launches0 = ipt.kernel_launch_count()
    orient_before = list(orient)
    torch.cuda.nvtx.range_push("timed")       # ncu --nvtx --nvtx-include "timed/"
    ev_first = args.steps - n_ev
    step_ev = []
    if flush is None:
        t_start.record()
        for s in range(args.steps):
            one_step(evs[s - ev_first] if s >= ev_first else None)
        t_end.record()
    else:   # L2-resident workload: L2 overwritten (read flush) before every step
        step_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(args.steps)]
        for s in range(args.steps):
            flush.sum()
            step_ev[s][0].record()
            one_step(evs[s - ev_first] if s >= ev_first else None)
            step_ev[s][1].record()
    last = t_end if flush is None else step_ev[-1][1]
    t_poll = 0.0
    while not last.query():   # clocks sampled while the GPU runs the timed steps
        if hasattr(clocks, "sample") and time.perf_counter() - t_poll > 0.002:
            clocks.sample()
            t_poll = time.perf_counter()
        time.sleep(0.0005)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
    launches = ipt.kernel_launch_count() - launches0
    clk = clocks.stop()
    elapsed_ms = t_start.elapsed_time(t_end) if flush is None else sum(a.elapsed_time(b) for a, b in step_ev)
    flushed = flush is not None
    del flush
    part.barrier()
    elapsed_ms = part.max_over_ranks(elapsed_ms, red_dev)

    # ---- throughput: whole-job bytes over the slowest rank's device time
    if sh is not None:
        job_bytes = sh.job_bytes_per_step()
    else:
        job_bytes = world * sum(2 * M * N * eb for (_, M, N, _, _) in mats)
    value_gbs = part.aggregate_gbs(job_bytes, args.steps, elapsed_ms)
    peak, peak_src = load_peaks()

    # ---- per-stage (per-kernel) live timing on the last two steps -> roofline
    kern = {}          # name -> [ms, bytes, launches]
    per_shape = {}
    S_bytes = 0        # stage-scaled bytes of the timed steps (this rank)
    orient_sim = list(orient_before)
    for s in range(args.steps):
        timed = s >= ev_first
        for i, (t, M, N, cnt, _) in enumerate(mats):
            if cnt == 0:
                continue
            a, b = (M, N) if fixed else ((N, M) if orient_sim[i] else (M, N))
            p = plans[(a, b)]
            S_bytes += 2 * a * b * eb * cnt * p.n_stages
            if timed:
                ms = [evs[s - ev_first][i][st].elapsed_time(evs[s - ev_first][i][st + 1]) for st in range(3)]
                rec = _stage_rec(ipt, p, cnt, t, a, b, eb, ms)
                per_shape[f"{a}x{b}"] = {"count": cnt, "m": p.m, "n": p.n, "S": p.n_stages,
                                         "eff_gbs": round(2 * a * b * eb * cnt / (sum(ms) / 1e3) / 1e9, 1),
                                         "stages": rec}
                for r in rec:
                    k = kern.setdefault(r["kernel"], [0.0, 0, 0])
                    k[0] += r["ms"]
                    k[1] += 2 * a * b * eb * cnt
                    k[2] += 1
            orient_sim[i] = not orient_sim[i]
    local_ms = elapsed_ms   # max over ranks: the stage-scaled fraction of the slowest rank
    stage_scaled = part.sum_over_ranks(S_bytes, red_dev) / (local_ms / 1e3) / 1e9 / peak
    roofline = None
    if kern:
        dom = max(kern, key=lambda k: kern[k][0])
        kms, kb, kn = kern[dom]
        achieved = kb / (kms / 1e3) / 1e9
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            try:
                traffic = json.load(open(tp)).get(args.workload, {}).get(dom)
            except Exception:
                traffic = None
        ev_ms = sum(sum(evs[j][i][0].elapsed_time(evs[j][i][3]) for i in range(len(mats)) if mats[i][3])
                    for j in range(n_ev))
        roofline = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": peak,
                    "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                    "peak_source": peak_src, "launches": kn, "avg_launch_ms": round(kms / kn, 4),
                    "share_of_step": round(kms / ev_ms, 4) if ev_ms else None,
                    "algorithmic_bytes_per_launch": kb // kn,
                    "stage_events": f"last {n_ev} of {args.steps} timed steps" + ("" if fixed else " (both orientations)"),
                    "per_kernel": {k: {"ms": round(v[0], 3), "gbs": round(v[1] / (v[0] / 1e3) / 1e9, 1),
                                       "launches": v[2]} for k, v in kern.items()}}

    # ---- the reverse shape (N x M) for context: two untimed steps with stage events
    per_shape_rev = {}
    if fixed and sh is not None and sh.count:
        for _ in range(2):
            ev_r = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in mats]
            one_step(ev_r, reverse=True)
            torch.cuda.synchronize()
            for i, (t, M, N, cnt, _) in enumerate(mats):
                ms = [ev_r[i][st].elapsed_time(ev_r[i][st + 1]) for st in range(3)]
                p = plans[(N, M)]
                per_shape_rev[f"{N}x{M}"] = {"count": cnt, "m": p.m, "n": p.n, "S": p.n_stages,
                                             "eff_gbs": round(2 * M * N * eb * cnt / (sum(ms) / 1e3) / 1e9, 1),
                                             "stages": _stage_rec(ipt, p, cnt, t, N, M, eb, ms),
                                             "note": "untimed, not in value: the reverse shape for context"}

    # ---- verification of the final state (sampled definition check, every rank)
    ok = True
    for i, (t, M, N, cnt, t0) in enumerate(mats):
        if cnt:
            ok &= _verify(t, M, N, eb, False, t0=t0, count=cnt, seed=i, seq=seqs[i])
    ok = part.all_ok(ok, red_dev)
    for m in mats:
        m[0] = None
    mats.clear()
    torch.cuda.empty_cache()

    # ---- e2e through the public host API (H2D + stages + D2H; Sec. 6)
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, ipt, torch, dev, red_dev, part, wl, sh, world, rank)

    # ---- sub-records: every other BASELINE config (N = 1 only)
    subs = {}
    if world == 1 and args.sub != "none":
        names = SUB_ORDER if args.sub == "all" else [x for x in args.sub.split(",") if x]
        for name in names:
            if name == args.workload or name not in WORKLOADS:
                continue
            log(f"[bench] sub-record {name}")
            subs[name] = run_sub(ipt, torch, dev, name, args.sub_steps, 3, args.autotune)
            ok &= subs[name]["verified"]

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(wl)

    if rank == 0:
        plans_cfg = {f"{a}x{b}": {"m": p.m, "n": p.n, "S": p.n_stages,
                                  "variant": [ipt.VARIANTS[v] for v in p.variant]}
                     for (a, b), p in plans.items()}
        line = {
            "metric": METRIC, "value": round(value_gbs, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(elapsed_ms / args.steps, 4), "higher_is_better": True,
            "scaling": "strong" if sh is not None else "weak", "vs_baseline": None,
            "dtype": "u32" if eb == 4 else "u64", "data": "synthetic",
            "config": {"workload": wl["name"],
                       "shapes": [f"{M}x{N}" for (M, N) in wl["shapes"]],
                       "elem_bytes": eb, "batch": wl.get("batch", 1),
                       "per_rank": (f"matrices [{sh.lo}, {sh.hi}) of {sh.total} on rank 0"
                                    if sh is not None else "every matrix on every rank"),
                       "plans": plans_cfg,
                       "l2": ("no flush: the inputs exceed the 126 MB L2" if not flushed else
                              "L2 flushed before every step (512 MB read, outside the step's events)"),
                       "parallelism": (f"batch shards x{world} (no collective on the data path)"
                                       if sh is not None else f"replicas x{world}"),
                       "planning": (f"ipt_plan_autotune, {args.autotune} candidates per shape "
                                    "(before the timed region)") if args.autotune > 1 else "cost model",
                       "orientation": ("fixed: every step transposes the configured shape (the previous "
                                       "step's transposes re-read as the next inputs; final state checked "
                                       "against the composition of all transposes)" if fixed else
                                       "alternate: the configured shape and its transpose on alternate steps")},
            "hbm_frac_stage_scaled": round(stage_scaled, 4),
            "per_shape": per_shape, "per_shape_reverse": per_shape_rev or None,
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": launches, "clocks": clk, "verified": ok, "sub": subs,
        }
        emit(line, args)
    part.barrier()
    if world > 1:
        import torch.distributed as dist

        dist.destroy_process_group()
    return 0 if ok else 1


def run_e2e(args, ipt, torch, dev, red_dev, part, wl, sh, world, rank):
    """The same metric end to end through the public host API: every step copies the
    step's inputs from pinned host memory to the device, transposes them and copies the
    results back (ipt_transpose_host_pipeline: H2D of matrix i+1 and D2H of matrix i-1
    overlap the stages of matrix i).  At N = 1 also the paper's synchronous vs
    asynchronous comparison (Sec. 6)."""
    from inputs import seeded

    eb = wl["eb"]
    tdt = torch.int32 if eb == 4 else torch.int64
    if sh is not None:
        M, N = sh.M, sh.N
        cnt = min(sh.count, args.e2e_count)
        shapes = [(M, N)] * cnt
        t0s = [sh.lo + i for i in range(cnt)]
    else:
        shapes = list(wl["shapes"])
        t0s = [0] * len(shapes)
    hosts = []
    for (M, N), t0 in zip(shapes, t0s):
        h = torch.empty(M * N, dtype=tdt, pin_memory=True)
        tmp = torch.empty(M * N, dtype=tdt, device=dev)
        seeded.fill_device_(tmp, M, N, eb, t0=t0)
        h.copy_(tmp)
        hosts.append([h, M, N, False])
    del tmp
    torch.cuda.synchronize()

    def pipe_step():
        cur = [(N, M) if tr else (M, N) for (_, M, N, tr) in hosts]
        if hosts:
            ipt.transpose_host_pipeline_([h for (h, _, _, _) in hosts], cur)
        for hm in hosts:
            hm[3] = not hm[3]

    pipe_step()   # warm-up (allocates the device slots)
    torch.cuda.synchronize()
    part.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    w0 = time.perf_counter()
    e0.record()
    for _ in range(args.e2e_steps):
        pipe_step()
    e1.record()
    torch.cuda.synchronize()
    wall = time.perf_counter() - w0
    ms = part.max_over_ranks(e0.elapsed_time(e1), red_dev)
    hb = sum(M * N * eb for (_, M, N, _) in hosts)
    job = part.sum_over_ranks(hb, red_dev)
    ok = True
    h, M, N, tr = hosts[0]
    idx = torch.randint(0, M * N, (2048,))
    src = (idx % M) * N + idx // M if tr else idx
    ok &= bool(torch.equal(h[idx], seeded.values_torch_sample(src + t0s[0] * M * N, eb).to(h.dtype)))
    out = {"value": round(2 * job * args.e2e_steps / (ms / 1e3) / 1e9, 3), "unit": "GB/s",
           "h2d_bytes_per_step": hb, "d2h_bytes_per_step": hb, "steps": args.e2e_steps,
           "matrices_per_rank": len(hosts), "wall_s": round(wall, 3), "verified": ok,
           "api": "ipt_transpose_host_pipeline (pinned host buffers; H2D of matrix i+1 and D2H of "
                  "matrix i-1 overlap the stages of matrix i)"}
    if world == 1 and hosts:
        # E10: synchronous (Q = 1: H2D, stages, D2H in sequence) vs the
        # asynchronous schemes, on the first 16 matrices
        sub = hosts[:16]
        modes = {}
        for mode in ("sync_q1", "async_q4", "pipeline"):
            def step():
                if mode == "pipeline":
                    ipt.transpose_host_pipeline_([h for (h, _, _, _) in sub],
                                                 [(N, M) if tr else (M, N) for (_, M, N, tr) in sub])
                else:
                    for (h, M, N, tr) in sub:
                        a, b = (N, M) if tr else (M, N)
                        ipt.transpose_host_(h, a, b, queues=1 if mode == "sync_q1" else 4)
                for hm in sub:
                    hm[3] = not hm[3]
            step()
            torch.cuda.synchronize()
            a0 = time.perf_counter()
            for _ in range(2):
                step()
            torch.cuda.synchronize()
            dt = time.perf_counter() - a0
            modes[mode] = round(2 * 2 * sum(M * N * eb for (_, M, N, _) in sub) / dt / 1e9, 2)
        out["sync_vs_async"] = dict(modes, matrices=len(sub), unit="GB/s (host wall clock)",
                                    note="sync_q1 = ipt_transpose_host queues=1 per matrix; async_q4 = "
                                         "stages 2-3 + D2H split over 4 queues per matrix (Fig. 5b); "
                                         "pipeline = across matrices")
    for hm in hosts:
        hm[0] = None
    hosts.clear()
    return out


def cpu_baseline(wl):
    """The oracle as it stands on the host cores, bounded: for C5 one matrix per core
    (embarrassingly parallel), plus one matrix on one thread."""
    eb = wl["eb"]
    M, N = wl["shapes"][0]
    cores = min(host_cores(), 64)
    b1, t1 = oracle_single(M, N, eb)
    out = {"unit": "GB/s", "kind": "oracle", "cpu_model": cpu_model(), "host_cpus": os.cpu_count(),
           "single_thread": round(b1 / t1 / 1e9, 4)}
    if "batch" in wl:
        b, t, cpu_s = oracle_per_core(M, N, eb, 0, cores)
        out.update(value=round(b / t / 1e9, 4), cores=cores,
                   sample=f"{cores} {M}x{N} matrices of the batch, one per host thread "
                          f"({cpu_s:.1f} s of CPU work); single_thread = one matrix on one thread")
    else:
        out.update(value=out["single_thread"], cores=1, sample=f"one {M}x{N} matrix, one thread")
    return out


if __name__ == "__main__":
    sys.exit(main())
