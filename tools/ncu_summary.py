"""Summarise ncu reports (.ncu-rep) and launch lists into profiles/ (markdown + json).

    python tools/ncu_summary.py OUT_PREFIX rep1.ncu-rep [rep2 ...] [--launches launches.csv]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_pct"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_pct"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_pct"),
    ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "fp64_pipe_pct"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "alu_pipe_pct"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "fma_pipe_pct"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem_wavefronts"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__shared_mem_per_block_dynamic", "dyn_smem"),
    ("sm__inst_executed.sum", "inst_executed"),
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 2:
        return []
    h, units = rows[0], rows[1]
    res = []
    for v in rows[2:] if len(rows) > 2 else rows[1:]:
        d = {"kernel": v[h.index("Kernel Name")] if "Kernel Name" in h else "?"}
        for k, name in KEYS:
            if k in h:
                i = h.index(k)
                try:
                    d[name] = float(v[i].replace(",", ""))
                except ValueError:
                    d[name] = v[i]
                d[name + "_unit"] = units[i]
        stalls = []
        for i, c in enumerate(h):
            if c.startswith("smsp__average_warps_issue_stalled_") and c.endswith("per_issue_active.ratio"):
                try:
                    stalls.append((float(v[i]), c.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")))
                except ValueError:
                    pass
        d["top_stalls"] = [(n, round(x, 3)) for x, n in sorted(stalls, reverse=True)[:5]]
        res.append(d)
    return res


def to_bytes(v, unit):
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


def to_us(v, unit):
    return v * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3, "second": 1e6}.get(unit, 1)


def main():
    args = sys.argv[1:]
    launches = None
    dominant = None
    if "--dominant" in args:                 # --dominant PATTERN KERNEL_SUBSTRING
        i = args.index("--dominant")
        dominant = (args[i + 1], args[i + 2])
        args = args[:i] + args[i + 3:]
    if "--launches" in args:
        i = args.index("--launches")
        launches = args[i + 1]
        args = args[:i] + args[i + 2:]
    prefix, reps = args[0], args[1:]
    summary = {"kernels": []}
    md = ["| kernel | us | DRAM read MB | DRAM write MB | DRAM % | SM % | issue % | warps % | FP64 pipe % | regs | top stalls |",
          "|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in reps:
        for d in raw(rep):
            us = to_us(d.get("duration", 0), d.get("duration_unit", ""))
            rd = to_bytes(d.get("dram_read", 0), d.get("dram_read_unit", ""))
            wr = to_bytes(d.get("dram_write", 0), d.get("dram_write_unit", ""))
            d["duration_us"], d["dram_read_bytes"], d["dram_write_bytes"] = us, rd, wr
            summary["kernels"].append(d)
            name = d["kernel"].split("(")[0][:40]
            md.append(f"| {name} | {us:.1f} | {rd/1e6:.1f} | {wr/1e6:.1f} | {d.get('dram_pct', 0):.1f} | "
                      f"{d.get('sm_pct', 0):.1f} | {d.get('issue_pct', 0):.1f} | {d.get('warps_active_pct', 0):.1f} | "
                      f"{d.get('fp64_pipe_pct', 0):.1f} | {int(d.get('regs', 0))} | "
                      f"{', '.join(f'{n} {x}' for n, x in d['top_stalls'][:3])} |")
    if launches:
        rows = list(csv.reader(open(launches)))
        hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[hdr_i]
        ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
        ui = h.index("Metric Unit") if "Metric Unit" in h else None
        agg = {}
        for r in rows[hdr_i + 1:]:
            if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
                continue
            v = float(r[vi].replace(",", ""))
            us = to_us(v, r[ui]) if ui is not None else v
            k = r[ki].split("(")[0]
            agg.setdefault(k, []).append(us)
        tot = sum(sum(v) for v in agg.values())
        summary["launches"] = {k: {"count": len(v), "mean_us": sum(v) / len(v), "share": sum(v) / tot} for k, v in agg.items()}
        md += ["", "Launch list (ncu gpu__time_duration, cold-cache, serialised):", "",
               "| kernel | launches | mean us | share of step |", "|---|---|---|---|"]
        for k, s in sorted(summary["launches"].items(), key=lambda kv: -kv[1]["share"]):
            md.append(f"| {k[:60]} | {s['count']} | {s['mean_us']:.1f} | {100 * s['share']:.1f}% |")
    if dominant:
        pat, sub = dominant
        ks = [k for k in summary["kernels"] if sub in k["kernel"]]
        if ks:
            k = ks[0]
            import os
            out = {"kernel_pattern": pat, "kernel": k["kernel"], "source": [prefix + ".json"], "reports": reps,
                   "dram_bytes_per_launch": k["dram_read_bytes"] + k["dram_write_bytes"],
                   "dram_read_bytes": k["dram_read_bytes"], "dram_write_bytes": k["dram_write_bytes"],
                   "duration_us_cold": k["duration_us"]}
            with open(os.path.join(os.path.dirname(prefix) or ".", "ncu_dominant.json"), "w") as f:
                json.dump(out, f, indent=1)
    with open(prefix + ".json", "w") as f:
        json.dump(summary, f, indent=1)
    with open(prefix + ".md", "w") as f:
        f.write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
