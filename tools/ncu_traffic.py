"""Per-kernel-class DRAM traffic of one bench step, measured by ncu WITHOUT cache
flushing between kernels (--cache-control none: L2 state as in the real step) and
without clock locking.  Writes profiles/<tag>_traffic.json, which bench.py reads for
roofline.traffic (bytes per launch of each sym_profile class).

    python tools/ncu_traffic.py <tag>      (on the GPU box)
"""
import csv
import json
import os
import re
import subprocess
import sys
from collections import OrderedDict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# ncu kernel names -> sym_profile kernel classes (the first matching prefix wins)
CLASSES = [("k_split_rand", "split_rand"), ("k_split<2", "split_degk"), ("k_split<0", "split_none"),
           ("k_split<1", "split_rand"),
           ("k_mis_round", "mis_round"), ("k_mis_huge", "mis_huge"), ("k_round0<0", "mis_round0"),
           ("k_round0<1", "mm_round0"), ("k_mm_round", "mm_round"), ("k_mm_huge", "mm_huge"),
           ("k_jpc_", "jp_build"), ("k_jp_rounds", "jp_rounds")]


def kclass(name):
    for pre, c in CLASSES:
        if name.startswith(pre):
            return c
    return None


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "run"
    out_csv = os.path.join(ROOT, "gpurun_out", f"{tag}_traffic.csv")
    os.makedirs(os.path.dirname(out_csv), exist_ok=True)
    cmd = ["ncu", "--cache-control", "none", "--clock-control", "none", "-k", "regex:^k_", "--metrics",
           "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors.sum,"
           "lts__throughput.avg.pct_of_peak_sustained_elapsed,dram__throughput.avg.pct_of_peak_sustained_elapsed",
           "--csv", "--log-file", out_csv,
           sys.executable, os.path.join(ROOT, "bench.py"), "--profile-only", "--steps", "1", "--warmup", "1"]
    subprocess.run(cmd, check=True, stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL, timeout=1800)
    rows = [l for l in open(out_csv) if l.startswith('"')]
    r = list(csv.reader(rows))
    h = r[0]
    ki, mi, ui, vi, ii = (h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Unit"),
                          h.index("Metric Value"), h.index("ID"))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
    per = OrderedDict()
    for x in r[1:]:
        name = re.sub(r"\(.*", "", x[ki]).replace("void ", "").replace("sym::", "").strip()
        per.setdefault(x[ii], {"name": name})[x[mi]] = float(x[vi].replace(",", "")) * scale.get(x[ui], 1.0)
    # libsym's launches only (graph generation is torch's); bench.py --profile-only
    # --warmup 1 --steps 1 runs the step twice: the second half is the measured step
    launches = [k for k in per.values() if kclass(k["name"]) is not None]
    step = launches[len(launches) // 2:]
    agg = OrderedDict()
    for k in step:
        c = kclass(k["name"])
        if c is None:
            continue
        a = agg.setdefault(c, {"launches": 0, "dram_bytes": 0.0, "us": 0.0, "kernels": set(), "l2_sectors": 0.0,
                               "l2_pct_us": 0.0, "dram_pct_us": 0.0})
        a["launches"] += 1
        t = k.get("gpu__time_duration.sum", 0.0)
        a["l2_sectors"] += k.get("lts__t_sectors.sum", 0.0)
        a["l2_pct_us"] += k.get("lts__throughput.avg.pct_of_peak_sustained_elapsed", 0.0) * t
        a["dram_pct_us"] += k.get("dram__throughput.avg.pct_of_peak_sustained_elapsed", 0.0) * t
        a["dram_bytes"] += k.get("dram__bytes_read.sum", 0.0) + k.get("dram__bytes_write.sum", 0.0)
        a["us"] += k.get("gpu__time_duration.sum", 0.0)
        a["kernels"].add(k["name"])
    classes = {c: {"launches": a["launches"], "dram_bytes": a["dram_bytes"],
                   "dram_bytes_per_launch": a["dram_bytes"] / a["launches"], "us": a["us"],
                   "l2_sectors": a["l2_sectors"],
                   # time-weighted ncu throughput fractions of the class (L2 = lts__throughput, the
                   # busiest L2 sub-unit; DRAM = dram__throughput)
                   "l2_frac": a["l2_pct_us"] / a["us"] / 100.0 if a["us"] else 0.0,
                   "dram_frac": a["dram_pct_us"] / a["us"] / 100.0 if a["us"] else 0.0,
                   "kernels": sorted(a["kernels"])} for c, a in agg.items()}
    res = {"tag": tag, "command": " ".join(cmd[:-7]) + " python bench.py --profile-only --steps 1 --warmup 1",
           "note": "DRAM bytes = dram__bytes_read.sum + dram__bytes_write.sum per kernel class over the measured "
                   "step (the second of two); serialised replay, no cache flush: compare shares and bytes, "
                   "not absolute times; l2_frac / dram_frac = time-weighted lts__throughput / dram__throughput "
                   "pct_of_peak_sustained_elapsed", "classes": classes}
    for dst in (os.path.join(ROOT, "profiles", f"{tag}_traffic.json"),
                os.path.join(ROOT, "gpurun_out", f"{tag}_traffic.json")):
        with open(dst, "w") as f:
            json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
