"""Print a compact summary of a bench.py JSON line (headline, roofline, e2e, sub-records).

    python tools/bench_summary.py gpurun_out/bench.json [--shapes]"""
import json
import sys
from collections import defaultdict

d = json.loads([x for x in open(sys.argv[1]).read().splitlines() if x.startswith("{")][-1])
show = "--shapes" in sys.argv
print("value", d["value"], d["unit"], "ms/step", d["ms_per_step"], "frac_S", d.get("hbm_frac_stage_scaled"),
      "launches", d.get("gpu_launches"), "verified", d.get("verified"))
print("clocks", d.get("clocks"))
r = d.get("roofline") or {}
print("roofline", r.get("kernel"), r.get("achieved"), r.get("frac"), r.get("per_kernel"))
print("per_shape", json.dumps(d.get("per_shape")))
e = d.get("e2e") or {}
print("e2e", e.get("value"), e.get("sync_vs_async"))
print("cpu", d.get("cpu_baseline"))
for name, s in (d.get("sub") or {}).items():
    print("==", name, s["value"], "sq", s.get("squares"), "rect", s.get("rectangles"), "ok", s["verified"], "wall", s["wall_s"])
    agg = defaultdict(lambda: [0.0, 0.0])
    for shp, rec in s["per_shape"].items():
        for o, stages in rec["stages"].items():
            M, N = map(int, o.split("x"))
            for x in stages:
                agg[x["kernel"]][0] += x["ms"]
                agg[x["kernel"]][1] += 2 * M * N * s["elem_bytes"]
        if show:
            st = {k: [(x["kernel"], x["gbs"]) for x in v] for k, v in rec["stages"].items()}
            print("   ", shp, rec["eff_gbs"], rec["plan"], st)
    tot = sum(v[0] for v in agg.values())
    print("    kernels:", ", ".join(f"{k} {v[0] / tot:.2f} @ {v[1] / v[0] / 1e6:.0f}" for k, v in
                                     sorted(agg.items(), key=lambda kv: -kv[1][0])))
