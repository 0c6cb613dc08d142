"""Per-kernel ncu table (one pipeline step) -> markdown: time, DRAM read/write bytes,
DRAM GB/s and its fraction of the measured HBM peak, L2 bytes.
    python tools/ncu_table.py <ncu.csv> <config> <out.md> [--append]
The CSV holds one graph launch (tools/prof_step.py, ncu --profile-from-start off)."""
import csv
import json
import os
import sys
from collections import OrderedDict

path, cfg, out = sys.argv[1:4]
append = "--append" in sys.argv
peak = 6455.3
try:
    peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                       "MEASURED_PEAKS.json")))["hbm_gbs"]
except Exception:
    pass
lines = open(path).read().splitlines()
i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
rows = list(csv.reader(lines[i:]))
h = rows[0]
per = OrderedDict()
for r in rows[1:]:
    if len(r) < len(h):
        continue
    kid = int(r[h.index("ID")])
    name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").split("::")[-1]
    d = per.setdefault(kid, {"name": name})
    v = r[h.index("Metric Value")].replace(",", "")
    unit = r[h.index("Metric Unit")]
    x = float(v)
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "usecond": 1e3, "msecond": 1e6}.get(unit, 1)
    d[r[h.index("Metric Name")]] = x * mult
ids = sorted(per)
ids = [k for k in ids if not per[k]["name"].startswith(("at::", "void at::"))]
step = ids  # one graph launch (prof_step.py brackets it with cudaProfilerStart/Stop)
agg = OrderedDict()
for k in step:
    d = per[k]
    a = agg.setdefault(d["name"], {"n": 0, "t": 0.0, "rd": 0.0, "wr": 0.0, "l2": 0.0})
    a["n"] += 1
    a["t"] += d.get("gpu__time_duration.sum", 0)
    a["rd"] += d.get("dram__bytes_read.sum", 0)
    a["wr"] += d.get("dram__bytes_write.sum", 0)
    a["l2"] += d.get("lts__t_bytes.sum", 0)
tt = sum(a["t"] for a in agg.values())
with open(out, "a" if append else "w") as f:
    if not append:
        f.write("# Per-kernel DRAM traffic (ncu), one pipeline step per config\n\n"
                "`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum "
                "--clock-control none` of `tools/prof_step.py <config>` (cold caches, serialised launches); "
                f"the graph launch's kernels. DRAM GB/s = (read + write) / duration; frac = that / {peak} GB/s "
                "(MEASURED_PEAKS.json). Low fractions on small, latency-bound launches are expected.\n")
    f.write(f"\n## {cfg}\n\n| kernel | launches | us | share | DRAM read MB | DRAM write MB | DRAM GB/s | frac of HBM | L2 MB |\n"
            "|---|---:|---:|---:|---:|---:|---:|---:|---:|\n")
    for name, a in sorted(agg.items(), key=lambda kv: -kv[1]["t"]):
        gbs = (a["rd"] + a["wr"]) / a["t"] if a["t"] else 0.0  # bytes / ns = GB/s
        f.write(f"| {name} | {a['n']} | {a['t'] / 1e3:.1f} | {a['t'] / tt:.1%} | {a['rd'] / 1e6:.1f} | "
                f"{a['wr'] / 1e6:.1f} | {gbs:.0f} | {gbs / peak:.3f} | {a['l2'] / 1e6:.1f} |\n")
    f.write(f"\n{sum(a['n'] for a in agg.values())} launches, {tt / 1e3:.1f} us in total.\n")
