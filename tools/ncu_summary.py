"""Summarise ncu captures into profiles/ (markdown + csv).

    python tools/ncu_summary.py <launches.csv> <full.ncu-rep> <out_prefix>

launches.csv: `ncu --metrics gpu__time_duration.sum --csv --log-file` of one bench
step (cold-cache, serialised: compare SHARES); full.ncu-rep: `ncu --set full` of the
top kernels.  Writes <out_prefix>_launches.csv (kernel class, launches, total us,
share) and <out_prefix>_ncu.md (per captured kernel: duration, DRAM bytes, DRAM /
L2 / SM throughput, occupancy, registers, top stall reasons).
"""
import csv
import re
import subprocess
import sys
from collections import OrderedDict


def launches(path):
    rows = [l for l in open(path) if l.startswith('"')]
    r = list(csv.reader(rows))
    h = r[0]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    agg = OrderedDict()
    for x in r[1:]:
        if x[mi] != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", x[ki]).replace("void ", "").replace("sym::", "").strip()
        if not name.startswith("k_"):  # graph generation (torch) is outside the step
            continue
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += float(x[vi].replace(",", "")) / 1000.0
    return agg


def full(path):
    out = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    r = list(csv.reader(out.splitlines()))
    h = r[0]
    units = dict(zip(h, r[1]))
    scale = {"byte": 1e-9, "Kbyte": 1e-6, "Mbyte": 1e-3, "Gbyte": 1.0, "Tbyte": 1e3}
    res = []
    for v in r[2:]:
        d = dict(zip(h, v))
        for key in ("dram__bytes_read.sum", "dram__bytes_write.sum"):  # -> GB
            try:
                d[key] = str(float(d[key].replace(",", "")) * scale.get(units.get(key, "Gbyte"), 1.0))
            except (KeyError, ValueError):
                pass
        tscale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "s": 1e6,
                  "second": 1e6}
        t_unit = units.get("gpu__time_duration.sum", "us")
        d["gpu__time_duration.sum"] = str(float(d["gpu__time_duration.sum"].replace(",", "")) * tscale.get(t_unit, 1.0))
        stalls = []
        for k, val in d.items():
            if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued"):
                try:
                    stalls.append((float(val.replace(",", "")), k[len("smsp__pcsamp_warps_issue_stalled_"):]))
                except ValueError:
                    pass
        tot = sum(s[0] for s in stalls) or 1.0
        top = ", ".join(f"{n} {s / tot * 100:.0f}%" for s, n in sorted(stalls, reverse=True)[:4])

        def f(k):
            try:
                return float(d.get(k, "nan").replace(",", ""))
            except ValueError:
                return float("nan")
        res.append({
            "kernel": re.sub(r"\(.*", "", d["Kernel Name"]).replace("void ", "").strip(),
            "grid": d.get("launch__grid_size"), "regs": d.get("launch__registers_per_thread"),
            "dur_us": f("gpu__time_duration.sum"),
            "dram_rd": f("dram__bytes_read.sum"), "dram_wr": f("dram__bytes_write.sum"),
            "dram_pct": f("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
            "lts_pct": f("lts__throughput.avg.pct_of_peak_sustained_elapsed"),
            "sm_pct": f("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
            "issue_pct": f("sm__inst_issued.avg.pct_of_peak_sustained_active"),
            "occ": f("sm__warps_active.avg.pct_of_peak_sustained_active"), "stalls": top,
            "units": (d.get("dram__bytes_read.sum"), h),
        })
    return res


def main():
    lpath, fpath, prefix = sys.argv[1:4]
    agg = launches(lpath)
    total = sum(v[1] for v in agg.values())
    with open(prefix + "_launches.csv", "w") as f:
        f.write("kernel,launches,total_us,share\n")
        for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"{k},{n},{us:.1f},{us / total:.4f}\n")
    rows = [r for p in fpath.split(",") for r in full(p)]
    with open(prefix + "_ncu.md", "w") as f:
        f.write(f"# ncu --set full summary ({fpath.split('/')[-1]})\n\n")
        f.write("Captured under gpurun with `--clock-control none` (cold cache, serialised replay: compare "
                "shares, not absolutes).  DRAM bytes as reported by ncu (`dram__bytes_read.sum`, "
                "`dram__bytes_write.sum`).\n\n")
        f.write("| kernel | grid | regs | duration | DRAM read GB | DRAM write GB | DRAM % | L2 % | SM % | issue % | "
                "occupancy % | top stalls |\n|---|---|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['kernel']} | {r['grid']} | {r['regs']} | {r['dur_us']:.1f} us | {r['dram_rd']:.3g} | "
                    f"{r['dram_wr']:.3g} | {r['dram_pct']:.1f} | {r['lts_pct']:.1f} | {r['sm_pct']:.1f} | "
                    f"{r['issue_pct']:.1f} | {r['occ']:.1f} | {r['stalls']} |\n")
        f.write("\n## Launch list of one bench step (shares)\n\n| kernel | launches | total us | share |\n|---|---|---|---|\n")
        for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"| {k} | {n} | {us:.1f} | {us / total * 100:.1f}% |\n")
    print(open(prefix + "_ncu.md").read())


if __name__ == "__main__":
    main()
