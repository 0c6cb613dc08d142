"""Summarise ncu outputs into profiles/ (run locally on the files gpurun brought back).

    python tools/ncu_summary.py launches <launches.csv> <out.md>
    python tools/ncu_summary.py full <report.ncu-rep> <out.md> [<traffic.json> <config>]
"""
import csv
import io
import json
import subprocess
import sys
from collections import OrderedDict, defaultdict


def launches(path, out):
    lines = open(path).read().splitlines()
    i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
    rows = list(csv.reader(lines[i:]))
    h = rows[0]
    per = []
    for r in rows[1:]:
        if len(r) < len(h):
            continue
        if r[h.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        per.append((int(r[h.index("ID")]), r[h.index("Kernel Name")], float(r[h.index("Metric Value")])))
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for _, n, t in per:
        key = n.split("(")[0].replace("void ", "").replace("gm::<unnamed>::", "")
        tot[key] += t
        cnt[key] += 1
    all_t = sum(tot.values())
    with open(out, "w") as f:
        f.write(f"# Launch list summary ({path})\n\n")
        f.write("ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised launches;\n"
                "compare SHARES, not absolute times, with bench.py's CUDA-event stage times).\n\n")
        f.write("| kernel | launches | total us | share |\n|---|---:|---:|---:|\n")
        for k in sorted(tot, key=lambda k: -tot[k]):
            f.write(f"| {k} | {cnt[k]} | {tot[k] / 1e3:.1f} | {tot[k] / all_t:.1%} |\n")
        f.write(f"\n{len(per)} launches, {all_t / 1e3:.1f} us total\n")


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "smsp__inst_executed.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "launch__grid_size", "launch__block_size"]


def full(path, out, traffic_json=None, config=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    with open(out, "w") as f:
        f.write(f"# ncu --set full summary ({path})\n\n")
        for r in rows[2:]:
            name = r[h.index("Kernel Name")]
            f.write(f"## {name[:120]}\n\n| metric | value | unit |\n|---|---:|---|\n")
            for w in WANT:
                if w in h:
                    f.write(f"| {w} | {r[h.index(w)]} | {units[h.index(w)]} |\n")
            tot = float(r[h.index("smsp__pcsamp_sample_count")].replace(",", "") or 1)
            f.write("\nStall reasons (share of PC samples):\n\n")
            st = []
            for i, c in enumerate(h):
                if c.startswith("smsp__pcsamp_warps_issue_stalled") and not c.endswith("not_issued"):
                    try:
                        v = float(r[i].replace(",", "") or 0)
                    except ValueError:
                        continue
                    if v / tot > 0.02:
                        st.append((v / tot, c.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            for v, c in sorted(st, reverse=True):
                f.write(f"- {c}: {v:.1%}\n")
            f.write("\n")
            if traffic_json and "k_find" in name:
                rd = float(r[h.index("dram__bytes_read.sum")].replace(",", ""))
                wr = float(r[h.index("dram__bytes_write.sum")].replace(",", ""))
                ur, uw = units[h.index("dram__bytes_read.sum")], units[h.index("dram__bytes_write.sum")]
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
                t = rd * scale[ur] + wr * scale[uw]
                try:
                    d = json.load(open(traffic_json))
                except Exception:
                    d = {}
                sec = float(r[h.index("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum")].replace(",", ""))
                d[config] = {"kernel": "k_find", "traffic_bytes": t, "l1_ld_sectors": sec, "source": path}
                json.dump(d, open(traffic_json, "w"), indent=1)


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        full(sys.argv[2], sys.argv[3], *(sys.argv[4:6] if len(sys.argv) > 5 else []))
