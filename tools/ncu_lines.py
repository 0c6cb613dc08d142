"""Per-source-line instruction/stall table from an ncu report (needs -lineinfo builds).
    python tools/ncu_lines.py report.ncu-rep [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname = None; hdr = None; agg = {}
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or len(r) < len(hdr): continue
    try:
        ie = int(r[hdr.index("Instructions Executed")] or 0); ss = int(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
    except ValueError:
        continue
    if r[0]:  # source line row carries the line's aggregate
        agg[(fname, int(r[0]))] = [ie, ss, r[1][:90]]
ti = sum(v[0] for v in agg.values()) or 1; ts = sum(v[1] for v in agg.values()) or 1
print(f"total instr {ti}  samples {ts}")
for k, v in sorted(agg.items(), key=lambda kv: -(kv[1][0] / ti + kv[1][1] / ts))[:top]:
    print(f"{k[0]}:{k[1]:4d} instr {100*v[0]/ti:5.1f}%  stall {100*v[1]/ts:5.1f}%  {v[2]}")
