"""Summarise ncu outputs from gpurun_out/ into committed profiles/ files.

    python tools/summarize_ncu.py <round tag, e.g. r01>

Reads gpurun_out/launches.csv (launch list of `bench.py --steps 2 --warmup 3`, metrics
gpu__time_duration.sum + dram bytes) and gpurun_out/prof_*.ncu-rep (full captures), writes
profiles/<tag>_launches.md, profiles/<tag>_ncu_full.md and profiles/traffic.json (per-launch
DRAM traffic of each libipt kernel kind, read by bench.py for the roofline 'traffic' key).
"""
import csv
import json
import os
import re
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GO = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
NCU = "/usr/local/cuda/bin/ncu"


def kind(name: str):
    """Kernel family as bench.py names it: cycle_global, or tile_onchip for every tile-stage
    kernel (tile_onchip_*, tile_group_db, tile_group_generic, tile_generic_cluster)."""
    if "cycle_global" in name or "cycle_ua" in name or "cycle_seg" in name:
        return "cycle_global"
    if "tile_" in name:
        return "tile_onchip"
    if "square_swap" in name:
        return "square_swap"
    return None


def launches(tag, workload="sweep"):
    path = os.path.join(GO, "launches.csv" if workload == "sweep" else f"launches_{workload}.csv")
    if not os.path.exists(path):
        return
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    idx = {h: i for i, h in enumerate(hdr)}
    per = defaultdict(dict)
    for r in rows[1:]:
        lid = int(r[idx["ID"]])
        per[lid]["name"] = r[idx["Kernel Name"]]
        v = float(r[idx["Metric Value"]].replace(",", ""))
        m = r[idx["Metric Name"]]
        unit = r[idx["Metric Unit"]]
        if m == "gpu__time_duration.sum":
            v = v / 1e3 if unit in ("ns", "nsecond") else (v if unit in ("us", "usecond") else v * 1e3)
            per[lid]["us"] = v
        elif m.startswith("dram__bytes"):
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(unit, 1)
            per[lid][m] = v * scale
    agg = defaultdict(lambda: {"n": 0, "us": 0.0, "rd": 0.0, "wr": 0.0})
    for lid, d in per.items():
        k = kind(d["name"])
        if k is None:
            continue
        a = agg[k]
        a["n"] += 1
        a["us"] += d.get("us", 0.0)
        a["rd"] += d.get("dram__bytes_read.sum", 0.0)
        a["wr"] += d.get("dram__bytes_write.sum", 0.0)
    tot = sum(a["us"] for a in agg.values())
    cmd = "python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu" + ("" if workload == "sweep" else f" --workload {workload}")
    lines = [f"# {tag}: ncu launch list of `{cmd}`",
             "", "Cold-cache, serialised (`--clock-control none`); compare SHARES, not absolutes. "
             "Only libipt kernels are aggregated (torch generator fills run outside the timed region).",
             "", "| kernel | launches | total µs | share | avg µs/launch | DRAM read MB/launch | DRAM write MB/launch |",
             "|---|---|---|---|---|---|---|"]
    traffic = {}
    for k, a in sorted(agg.items()):
        lines.append(f"| {k} | {a['n']} | {a['us']:.1f} | {a['us'] / tot:.3f} | {a['us'] / a['n']:.1f} | "
                     f"{a['rd'] / a['n'] / 1e6:.1f} | {a['wr'] / a['n'] / 1e6:.1f} |")
        traffic[k] = round((a["rd"] + a["wr"]) / a["n"])
    suffix = "" if workload == "sweep" else f"_{workload}"
    open(os.path.join(PROF, f"{tag}_launches{suffix}.md"), "w").write("\n".join(lines) + "\n")
    tp = os.path.join(PROF, "traffic.json")
    cur = json.load(open(tp)) if os.path.exists(tp) else {}
    cur[workload] = traffic
    cur["_note"] = ("bytes per launch (dram read + write), averaged over the libipt launches of "
                    "each workload's bench under ncu; source: profiles/%s_launches*.md" % tag)
    json.dump(cur, open(tp, "w"), indent=1)
    print("\n".join(lines))


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size",
        "launch__block_size", "lts__t_requests_op_atom.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "smsp__inst_executed.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_st.sum",
        "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum"]


def full(tag):
    out = [f"# {tag}: ncu --set full captures (`tools/prof_one.py 12800 15000`, 9998 12288, "
           "16384 16384 for square_swap, 20000 30000 f64 for cycle_seg)", ""]
    for rep in sorted(f for f in os.listdir(GO) if f.startswith("prof_") and f.endswith(".ncu-rep")):
        raw = subprocess.run([NCU, "-i", os.path.join(GO, rep), "--page", "raw", "--csv"],
                             capture_output=True, text=True).stdout
        rows = list(csv.reader(raw.splitlines()))
        if len(rows) < 3:
            continue
        hdr, units = rows[0], rows[1]
        for row in rows[2:]:
            d = dict(zip(hdr, row))
            u = dict(zip(hdr, units))
            out.append(f"## {rep}: `{d.get('Kernel Name', '?')[:90]}`")
            out.append("")
            out.append("| metric | value | unit |")
            out.append("|---|---|---|")
            for w in WANT:
                if w in d:
                    out.append(f"| {w} | {d[w]} | {u.get(w, '')} |")
            def num(k):
                try:
                    return float(d.get(k, "").replace(",", ""))
                except ValueError:
                    return None
            for op in ("ld", "st"):
                sec = num(f"l1tex__t_sectors_pipe_lsu_mem_global_op_{op}.sum")
                req = num(f"l1tex__t_requests_pipe_lsu_mem_global_op_{op}.sum")
                if sec and req:
                    out.append(f"| global {op} sectors / request (LSU; TMA copies not counted) | {sec / req:.2f} | |")
            stalls = sorted(((float(d[h].replace(',', '') or 0), h) for h in hdr
                             if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued")
                             and re.match(r"^[0-9.,]+$", d[h] or "x")), reverse=True)[:6]
            out.append("")
            out.append("Top stall reasons (pc samples): " + ", ".join(
                f"{h.replace('smsp__pcsamp_warps_issue_stalled_', '')}={int(v)}" for v, h in stalls))
            out.append("")
    open(os.path.join(PROF, f"{tag}_ncu_full.md"), "w").write("\n".join(out) + "\n")
    print("\n".join(out)[:4000])


if __name__ == "__main__":
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    os.makedirs(PROF, exist_ok=True)
    for w in ("sweep", "c1", "c3", "c4", "c5"):
        launches(tag, w)
    full(tag)
