"""Hottest SASS instructions of an ncu report (source page, --set full, -lineinfo):
    python tools/ncu_hot.py rep.ncu-rep [N]
prints the N instructions with the most warp-stall samples, their share, and the two
largest stall reasons of each (neighbouring instructions give the source context)."""
import csv
import io
import subprocess
import sys

rep, n = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
lines = out.splitlines()
i = [k for k, l in enumerate(lines) if l.startswith('"Address"')][0]
rows = list(csv.reader(io.StringIO("\n".join(lines[i:]))))
h = rows[0]
si = h.index("Warp Stall Sampling (All Samples)")
stall = [k for k, x in enumerate(h) if x.startswith("stall_") or "Stall" in x and k > si + 1]
tot = sum(float(r[si] or 0) for r in rows[1:] if len(r) == len(h))
body = [r for r in rows[1:] if len(r) == len(h)]
idx = sorted(range(len(body)), key=lambda k: -float(body[k][si] or 0))[:n]
for k in sorted(idx):
    r = body[k]
    def num(x):
        try:
            return float(x)
        except ValueError:
            return None
    reasons = sorted(((num(r[c]), h[c]) for c in range(si + 2, len(h)) if h[c].startswith("stall_")
                      and "Not Issued" not in h[c] and num(r[c]) is not None), reverse=True)[:2]
    print(f"{k:6d} {float(r[si]) / tot * 100:5.1f}%  {r[1].strip()[:60]:60s} " +
          " ".join(f"{name}={v:.0f}" for v, name in reasons))
