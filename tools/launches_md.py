"""Summarise an ncu launch list of the C5 headline bench (gpurun_out/launches_c5.csv, the
`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv`
pass of tools/ncu_r02c.sh) into profiles/r02_launches_c5.md and the per-launch DRAM bytes
of profiles/traffic.json["c5"] (read by bench.py's roofline.traffic)."""
import collections
import csv
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3,
         "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3}


def main(timed=5):
    rows = list(csv.reader(open(os.path.join(ROOT, "gpurun_out", "launches_c5.csv"))))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hi]
    ci = {k: h.index(k) for k in ["ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"]}
    L = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) < len(h):
            continue
        d = L.setdefault(int(r[ci["ID"]]), {"name": r[ci["Kernel Name"]]})
        d[r[ci["Metric Name"]]] = float(r[ci["Metric Value"]].replace(",", "")) * SCALE.get(r[ci["Metric Unit"]], 1)
    ipt_l = [(k, v) for k, v in L.items() if "ipt::" in v["name"]]
    rev = ipt_l[-2:]              # the two untimed reverse-shape steps after the timed region
    ipt_l = ipt_l[:-2]
    last = ipt_l[-timed:]
    alg = 2 * 512 * 4096 * 3000 * 4 / 1e9
    out = ["# r02: ncu launch list of `python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub none --autotune 1` (C5 headline)", "",
           "Cold-cache, serialised (`--clock-control none`); the shares and per-launch DRAM bytes are what count, not",
           "absolute times. `--autotune 1` (the cost model's plan, the same plan the timed bench run's autotune picks:",
           "`config.plans` of `profiles/r02_bench.json`): under ncu's serialised replay the autotune timings are",
           "distorted (one capture picked a 2-stage plan). Earlier libipt launches are the plan-setup transposes.",
           f"The {timed} launches below are the 3 warm-up + 2 timed steps, every one a 4096x3000 -> 3000x4096",
           "transposition of the 512 matrices (row-split slices); the bench's two untimed reverse-shape steps",
           "(3000x4096, swizzled column slices) follow the table.", "",
           "| launch | kernel | µs | DRAM read GB | DRAM write GB | algorithmic GB (read+write) | DRAM / algorithmic |",
           "|---|---|---|---|---|---|---|"]
    tb = tt = 0.0
    for k, v in last:
        rd, wr, t = v["dram__bytes_read.sum"] / 1e9, v["dram__bytes_write.sum"] / 1e9, v["gpu__time_duration.sum"]
        tb += (rd + wr) * 1e9
        tt += t
        out.append(f"| {k} | `{v['name'][:60]}` | {t:.1f} | {rd:.3f} | {wr:.3f} | {alg:.3f} | {(rd + wr) / alg:.4f} |")
    for k, v in rev:
        rd, wr, t = v["dram__bytes_read.sum"] / 1e9, v["dram__bytes_write.sum"] / 1e9, v["gpu__time_duration.sum"]
        out.append(f"| {k} (reverse, untimed) | `{v['name'][:60]}` | {t:.1f} | {rd:.3f} | {wr:.3f} | {alg:.3f} | "
                   f"{(rd + wr) / alg:.4f} |")
    out += ["", f"tile_group_rf is 100 % of the timed step (one launch per step, 512 matrices). Per launch: "
            f"{tb / timed / 1e9:.3f} GB of DRAM traffic for {alg:.3f} GB algorithmic; average {tt / timed:.0f} µs "
            f"under ncu ({alg * 1e6 / (tt / timed):.0f} GB/s)."]
    c = collections.defaultdict(list)
    for k, v in ipt_l[:-timed]:
        c[v["name"].split("(")[0].replace("void ipt::", "")].append(v["gpu__time_duration.sum"])
    out += ["", "Other libipt launches before the timed region (µs per launch, 512 matrices): " +
            "; ".join(f"`{n}` {min(t):.0f}–{max(t):.0f}" for n, t in c.items())]
    open(os.path.join(ROOT, "profiles", "r02_launches_c5.md"), "w").write("\n".join(out) + "\n")
    tj = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
    tj["c5"] = {"tile_group_rf": int(tb / timed)}
    json.dump(tj, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1)
    print("\n".join(out))


if __name__ == "__main__":
    main()
