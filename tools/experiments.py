"""NEXT-F1: the paper's experiments re-run on synthetic stand-ins.

  fig4  extraction time vs |Q|: C4 reference, query prefixes, L = 50
  fig5  extraction time vs L: C4 pair, L in {20, 40, 50, 100, 150}
  fig7  load-balancing ablation: the tile scheduler vs a static
        one-lane-per-query-position schedule without redistribution or heavy spill,
        on C2/C3/C4 at several L
  tab34 index-build and extraction times per config (Table III/IV analogues, :230-258)

Times are CUDA-event device times of one pipeline (CUDA-graph) run per step (mean of
--steps after --warmup, L2 flushed before each step), per stage from the graph's
event nodes (pack R and pack Q run concurrently: the 'index' column includes both packs). Writes a JSON file and a
markdown summary. The paper's numbers are on a K20c with real genomes: context only.

    python tools/experiments.py --out profiles/r1_experiments [--steps 5]
"""
import argparse
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm, synth  # noqa: E402


def run(R_dev, Q_dev, L, ls, steps, warmup, q_range=None, opts=None):
    """The path as bench.py times it: one gpumem_pipeline_run per step (CUDA graph),
    stage times from the graph's own event nodes."""
    opts = opts or {}
    for k, v in opts.items():
        gm.set_option(k, v)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()
    gm.set_option("pipe_events", 1)  # stage times from event nodes (each costs a few us)
    pl = gm.Pipeline(R_dev.numel(), Q_dev.numel(), ls, L, q_range)  # captured with these options
    tot, prof_acc, n_mems = 0.0, {}, 0
    for i in range(warmup + steps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        pl.run(R_dev, Q_dev)
        b.record(stream)
        n_mems = pl.result()
        b.synchronize()
        if i >= warmup:
            tot += a.elapsed_time(b)
            for k, (t, _) in pl.profile().items():
                prof_acc[k] = prof_acc.get(k, 0.0) + t
    pl.free()
    for k in opts:
        gm.set_option(k, {"find_spill": 64, "static_lb": 0}.get(k, 0))
    stage = {k: v / steps for k, v in prof_acc.items()}
    index_ms = sum(v for k, v in stage.items() if k.startswith("index") or k == "pack")
    extract_ms = sum(v for k, v in stage.items() if k.startswith("find") or k == "sort")
    return {"ms": tot / steps, "mems": n_mems, "index_ms": index_ms, "extract_ms": extract_ms, "stage_ms": stage}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="profiles/r1_experiments")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    args = ap.parse_args()
    res = {"device": torch.cuda.get_device_name(0), "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())}
    c4 = synth.make_pair("c4")
    R4, Q4 = torch.from_numpy(c4.R).cuda(), torch.from_numpy(c4.Q).cuda()
    nQ = len(c4.Q)

    res["fig4"] = []
    for frac in (0.2, 0.4, 0.6, 0.8, 1.0):
        qn = int(nQ * frac)
        r = run(R4, Q4[:qn].contiguous(), 50, 13, args.steps, args.warmup)
        r.update(q_bp=qn)
        res["fig4"].append(r)
        print("fig4", qn, r["ms"], r["mems"], flush=True)

    res["fig5"] = []
    for L in (20, 40, 50, 100, 150):
        r = run(R4, Q4, L, 13, args.steps, args.warmup)
        r.update(L=L)
        res["fig5"].append(r)
        print("fig5", L, r["ms"], r["mems"], flush=True)

    res["fig7"] = []
    pairs = [("c2", None), ("c3", None), ("c4", c4)]
    for name, P in pairs:
        P = P or synth.make_pair(name)
        Rd, Qd = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
        for L in sorted({P.L, 30 if P.ls <= 13 else P.L, 100}):
            if L < P.ls:
                continue
            on = run(Rd, Qd, L, P.ls, args.steps, args.warmup)
            off = run(Rd, Qd, L, P.ls, args.steps, args.warmup, opts={"static_lb": 1, "find_spill": 1 << 30})
            assert on["mems"] == off["mems"]
            res["fig7"].append({"config": name, "L": L, "lb_ms": on["ms"], "static_ms": off["ms"],
                                "lb_extract_ms": on["extract_ms"], "static_extract_ms": off["extract_ms"],
                                "speedup_extract": off["extract_ms"] / max(on["extract_ms"], 1e-9), "mems": on["mems"]})
            print("fig7", name, L, on["extract_ms"], off["extract_ms"], flush=True)
        del Rd, Qd

    res["tab34"] = []
    for name in ("c1", "c2", "c3", "c4", "c5_l20", "c5_l50", "c5_l300"):
        P = synth.make_pair(name) if not name.startswith("c5") and name != "c4" else c4
        L, ls = synth.CONFIG_PARAMS[name]
        Rd, Qd = (R4, Q4) if P is c4 else (torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda())
        r = run(Rd, Qd, L, ls, args.steps, args.warmup)
        r.update(config=name, R_bp=len(P.R), Q_bp=len(P.Q), L=L, ls=ls,
                 q_mbps=len(P.Q) / 1e6 / (r["ms"] / 1e3), mems_per_s=r["mems"] / (r["ms"] / 1e3))
        res["tab34"].append(r)
        print("tab34", name, r["ms"], r["mems"], flush=True)

    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    json.dump(res, open(args.out + ".json", "w"), indent=1)
    with open(args.out + ".md", "w") as f:
        f.write(f"# Paper-experiment analogues on synthetic data ({res['device']}, {res['when']})\n\n")
        f.write("Device times (CUDA events, L2 flushed per step), mean of %d steps. Index = pack + index "
                "stages, extraction = find + sort stages.\n\n" % args.steps)
        f.write("## Fig. 4 analogue: time vs |Q| (C4 reference, query prefixes, L = 50)\n\n"
                "| Q Mbp | step ms | extraction ms | MEMs |\n|---:|---:|---:|---:|\n")
        for r in res["fig4"]:
            f.write(f"| {r['q_bp'] / 1e6:.1f} | {r['ms']:.3f} | {r['extract_ms']:.3f} | {r['mems']} |\n")
        f.write("\n## Fig. 5 analogue: time vs L (C4 pair)\n\n| L | step ms | index ms | extraction ms | MEMs |\n"
                "|---:|---:|---:|---:|---:|\n")
        for r in res["fig5"]:
            f.write(f"| {r['L']} | {r['ms']:.3f} | {r['index_ms']:.3f} | {r['extract_ms']:.3f} | {r['mems']} |\n")
        f.write("\n## Fig. 7 analogue: load balancing (tile scheduler vs static lane-per-position, no spill)\n\n"
                "| config | L | extraction ms (LB) | extraction ms (static) | speedup | MEMs |\n"
                "|---|---:|---:|---:|---:|---:|\n")
        for r in res["fig7"]:
            f.write(f"| {r['config']} | {r['L']} | {r['lb_extract_ms']:.3f} | {r['static_extract_ms']:.3f} | "
                    f"{r['speedup_extract']:.2f}x | {r['mems']} |\n")
        f.write("\n## Table III/IV analogue: index and extraction per config\n\n"
                "| config | R Mbp | Q Mbp | L | ls | index ms | extraction ms | step ms | Q Mbp/s | MEMs | MEMs/s |\n"
                "|---|---:|---:|---:|---:|---:|---:|---:|---:|---:|---:|\n")
        for r in res["tab34"]:
            f.write(f"| {r['config']} | {r['R_bp'] / 1e6:.2f} | {r['Q_bp'] / 1e6:.2f} | {r['L']} | {r['ls']} | "
                    f"{r['index_ms']:.3f} | {r['extract_ms']:.3f} | {r['ms']:.3f} | {r['q_mbps']:.0f} | "
                    f"{r['mems']} | {r['mems_per_s']:.3g} |\n")
    print("wrote", args.out)


if __name__ == "__main__":
    main()
