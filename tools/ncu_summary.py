"""Summarise an ncu --set full report: speed-of-light, FP64 pipe, DRAM bytes, occupancy, top stall
reasons and instruction mix. Usage: python tools/ncu_summary.py report.ncu-rep [--json out.json --key C3]"""
import csv
import io
import json
import subprocess
import sys
from collections import Counter


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0,
             "s": 1e3, "second": 1e3}
    recs = []
    for r in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, r):
            try:
                d[h] = float(v.replace(",", "")) * scale.get(u, 1.0)
            except ValueError:
                d[h] = v
        recs.append(d)
    return recs


def by_line(rep, top=25):
    """Stall samples aggregated by CUDA source line (cuda,sass view)."""
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows


def sass_mix(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Source" in r and "Address" in r)
    hdr = rows[hi]
    ix = {h: i for i, h in enumerate(hdr)}
    ex, st = Counter(), Counter()
    for r in rows[hi + 1:]:
        if len(r) < len(hdr):
            continue
        op = r[ix["Source"]].strip().split()
        if not op:
            continue
        o = op[1] if op[0].startswith("@") else op[0]
        o = o.split(".")[0]
        ex[o] += float(r[ix["Instructions Executed"]] or 0)
        st[o] += float(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    return ex, st


KEYS = {
    "duration_ms": ("gpu__time_duration.sum", 1),
    "fp64_pipe_pct": ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "inst_fp64_pct": ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", 1),
    "issue_active_pct": ("sm__inst_issued.avg.pct_of_peak_sustained_active", 1),
    "dram_read_bytes": ("dram__bytes_read.sum", 1),
    "dram_write_bytes": ("dram__bytes_write.sum", 1),
    "dram_pct": ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "l2_hit_pct": ("lts__t_sector_hit_rate.pct", 1),
    "warps_active": ("sm__warps_active.avg.per_cycle_active", 1),
    "regs": ("launch__registers_per_thread", 1),
    "block": ("launch__block_size", 1),
    "grid": ("launch__grid_size", 1),
    "ipc": ("sm__inst_executed.avg.per_cycle_active", 1),
}


def main():
    rep = sys.argv[1]
    recs = raw(rep)
    d = recs[0]
    s = {}
    for k, (m, sc) in KEYS.items():
        v = d.get(m)
        s[k] = v * sc if isinstance(v, float) else v
    stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): v for k, v in d.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and isinstance(v, float)
              and not k.endswith("not_issued")}
    tot = sum(stalls.values()) or 1
    s["stalls_pct"] = {k: round(100 * v / tot, 1) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:8]}
    ex, st = sass_mix(rep)
    tex = sum(ex.values()) or 1
    s["inst_mix_pct"] = {k: round(100 * v / tex, 1) for k, v in ex.most_common(12)}
    s["kernel"] = d.get("Kernel Name")
    print(json.dumps(s, indent=1))
    if "--json" in sys.argv:
        out = sys.argv[sys.argv.index("--json") + 1]
        key = sys.argv[sys.argv.index("--key") + 1]
        try:
            allj = json.load(open(out))
        except Exception:
            allj = {}
        s["dram_bytes_per_launch"] = (s["dram_read_bytes"] or 0) + (s["dram_write_bytes"] or 0)
        if "--matrices" in sys.argv:  # matrices factored by the captured launch (grid / CTAs per matrix)
            nm = int(sys.argv[sys.argv.index("--matrices") + 1])
            s["matrices"] = nm
            s["dram_bytes_per_matrix"] = s["dram_bytes_per_launch"] / nm
        s["report"] = rep
        allj[key] = s
        json.dump(allj, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
