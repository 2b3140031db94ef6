"""Summarise an ncu capture (launch list + --set full report) into profiles/.

    python scripts/ncu_summary.py gpurun_out/<tag> <round-tag> [--key 16384x16384]

Writes profiles/<round-tag>_ncu.md (share of each kernel in the launch list, and the key
metrics of the captured jacobi_iter_kernel launches) and updates profiles/ncu_traffic.json,
which bench.py reads for the roofline "traffic" field (DRAM bytes per launch).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__shared_mem_per_block_dynamic", "dyn smem/block"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("sm__cycles_active.avg", "SM active cycles"),
    ("sm__cycles_elapsed.avg", "SM elapsed cycles"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy %"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
]

SCALE = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "Tbyte": 1e12}


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next((r for r in rows if "Kernel Name" in r), None)
    agg = collections.defaultdict(list)
    for r in rows:
        if hdr is None or len(r) != len(hdr) or r is hdr:
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            agg[d["Kernel Name"].split("(")[0]].append(float(d["Metric Value"]))
    return agg


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {}
        for m, _ in METRICS:
            if m in hdr:
                i = hdr.index(m)
                d[m] = (r[i], units[i])
        d["Kernel Name"] = r[hdr.index("Kernel Name")]
        res.append(d)
    return res


def to_bytes(v, u):
    return float(v.replace(",", "")) * SCALE.get(u, 1.0)


def main():
    src, tag = sys.argv[1], sys.argv[2]
    key = sys.argv[sys.argv.index("--key") + 1] if "--key" in sys.argv else "16384x16384"
    lines = [f"# ncu summary {tag} (source: {src})", ""]
    lp = os.path.join(src, "launches.csv")
    if os.path.exists(lp):
        agg = launches(lp)
        tot = sum(sum(v) for v in agg.values())
        lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, cold/serialised)", "",
                  "| kernel | launches | mean µs | share |", "|---|---|---|---|"]
        for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
            lines.append(f"| {k} | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {sum(v) / tot:.3f} |")
        lines.append("")
    rep = os.path.join(src, "prof.ncu-rep")
    traffic = None
    if os.path.exists(rep):
        res = raw(rep)
        lines += ["## `ncu --set full` capture of the dominant kernel", ""]
        for n, d in enumerate(res):
            lines.append(f"### launch {n}: {d['Kernel Name'][:80]}")
            for m, label in METRICS:
                if m in d:
                    lines.append(f"- {label} (`{m}`): {d[m][0]} {d[m][1]}")
            if "dram__bytes_read.sum" in d and "dram__bytes_write.sum" in d:
                b = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
                lines.append(f"- DRAM read+write per launch: {b:.4e} B")
                traffic = b if traffic is None else min(traffic, b)
            lines.append("")
    open(os.path.join(ROOT, "profiles", f"{tag}_ncu.md"), "w").write("\n".join(lines) + "\n")
    if traffic is not None:
        tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        d = json.load(open(tp)) if os.path.exists(tp) else {}
        d[key] = {"dram_bytes_per_launch": traffic, "source": f"profiles/{tag}_ncu.md"}
        json.dump(d, open(tp, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
