"""Summarise ncu --set full captures (gpurun_out/<name>.ncu-rep) into a markdown table.

    python tools/ncu_report.py <out.md> name[@k]:algorithmic_bytes:units:description ...

For each capture: duration, DRAM read / write against the algorithmic bytes (read + write
of every moved byte once), achieved GB/s, L2 atomic requests per unit (claims of the
PTTWAC protocol), shared-memory bank conflicts next to the source-level
"L1 Wavefronts Shared Excessive" (conflicts that actually cost wavefronts), warps active,
registers, and the top warp-stall reasons."""
import csv
import io
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NCU = "/usr/local/cuda/bin/ncu"


def sel(skip):
    """ncu import filter: the skip-th launch of a multi-launch capture (name@skip)."""
    return ["--launch-skip", str(skip), "--launch-count", "1"] if skip else []


def raw(rep, skip=0):
    out = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv", *sel(skip)], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    return {h[i]: (v[i], u[i]) for i in range(len(h))}


def excessive(rep, skip=0):
    out = subprocess.run([NCU, "-i", rep, "--page", "source", "--csv", "--print-source", "sass", *sel(skip)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    try:
        i = h.index("L1 Wavefronts Shared Excessive")
        j = h.index("L1 Wavefronts Shared")
    except ValueError:
        return None, None
    ex = tot = 0.0
    for r in rows[2:]:
        try:
            ex += float(r[i] or 0)
            tot += float(r[j] or 0)
        except (ValueError, IndexError):
            pass
    return ex, tot


def num(d, k, scale=1.0):
    try:
        v, u = d[k]
        x = float(v.replace(",", ""))
    except (KeyError, ValueError):
        return None
    mult = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "ms": 1e-3, "us": 1e-6, "ns": 1e-9,
            "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9}.get(u, 1.0)
    return x * mult / scale


def main():
    out, specs = sys.argv[1], sys.argv[2:]
    lines = ["| capture | kernel | time | DRAM read / write (GB) | algorithmic (GB) | achieved (GB/s, algorithmic) | "
             "L2 atomic req / unit | smem bank conflicts (excess wavefronts / all) | warps active | regs | top stalls |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    notes = []
    for spec in specs:
        name, alg, units, desc = spec.split(":", 3)
        base, _, skip = name.partition("@")   # name@k: the k-th launch of the capture
        skip = int(skip or 0)
        rep = os.path.join(ROOT, "gpurun_out", base + ".ncu-rep")
        if not os.path.exists(rep):
            continue
        d = raw(rep, skip)
        t = num(d, "gpu__time_duration.sum")
        rd, wr = num(d, "dram__bytes_read.sum"), num(d, "dram__bytes_write.sum")
        alg, units = float(alg), float(units)
        atom = num(d, "lts__t_requests_op_atom.sum")
        bc = (num(d, "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum") or 0) + \
             (num(d, "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum") or 0)
        ex, wtot = excessive(rep, skip)
        stalls = []
        for k, (v, _) in d.items():
            if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                try:
                    stalls.append((float(v), k.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        tot_st = sum(s for s, _ in stalls) or 1
        top = ", ".join(f"{n} {s / tot_st:.0%}" for s, n in stalls[:3])
        kname = d.get("Kernel Name", ("?", ""))[0].replace("|", "/")
        lines.append(
            f"| {name} ({desc}) | `{kname[:60]}` | {t * 1e6:.1f} µs | {rd / 1e9:.3f} / {wr / 1e9:.3f} | {alg / 1e9:.3f} | "
            f"{alg / t / 1e9:.0f} | {atom / units if (atom is not None and units) else 0:.2f} | "
            f"{bc:.3g} ({(ex or 0):.3g} / {(wtot or 0):.3g}) | {d.get('sm__warps_active.avg.pct_of_peak_sustained_active', ('?',))[0]} % | "
            f"{d.get('launch__registers_per_thread', ('?',))[0]} | {top} |")
    open(out, "w").write("\n".join(lines) + "\n" + "\n".join(notes))
    print("\n".join(lines))


if __name__ == "__main__":
    main()
