#!/usr/bin/env python3
"""Benchmark: GPUMEM's hot path on B200 -- query Mbp/s (and MEMs/s) incl. index build.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c4] [--impl ours|reference]

One step = the whole hot path over the configured pair,
with the ASCII R and Q already resident in HBM: pack R, pack Q, index R, find
every MEM (lookup, extension, canonical-seed rule, compaction), sort by (r, q);
for N > 1 also the NCCL gather to rank 0 and rank 0's merge kernel. L2 is
flushed (a 512 MB write, > 126 MB L2) before every step, outside the timed
events. `value` = |Q| / (mean step time, max over ranks) in Mbp/s.

--impl reference times the CPU oracle (oracle/, the only reference this paper
tier has) on the box's host cores, each step a bounded sample of the workload.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_abu_dolehkac14_b200 import synth  # noqa: E402

METRIC = "query Mbp/s incl. index build (MEM extraction, GPUMEM hot path)"
WORKLOAD_DESC = {
    "c1": "C1: 100 kbp random R, Q = R + 1% SNPs + planted repeats, L=20, ls=10",
    "c2": "C2: 5 Mbp vs 5 Mbp (~5% divergence), L=20, ls=12",
    "c3": "C3: 50 Mbp vs 50 Mbp with segmental duplications, L=50, ls=13",
    "c4": "C4: human-chromosome-scale synthetic pair 250 Mbp vs 150 Mbp, L=100, ls=13",
    "c5_l20": "C5: C4 pair at L=20, ls=13", "c5_l50": "C5: C4 pair at L=50, ls=13",
    "c5_l100": "C5: C4 pair at L=100, ls=13", "c5_l300": "C5: C4 pair at L=300, ls=13",
}
ORACLE_SAMPLE_BP = {"ours": 40_000_000, "reference": 40_000_000}  # same bounded sample in both legs


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c4", choices=sorted(WORKLOAD_DESC))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--no-d9", action="store_true")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks (NVML, during the timed region)
_REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
            0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
            0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


class ClockSampler:
    def __init__(self, index=0, period=0.005):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.period = period
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self.nv, self.err = None, repr(e)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in _REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if os.environ.get("GM_BENCH_NOCLK"):  # diagnostics: no sampler thread
            self.nv = None
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ CPU oracle timing (cpu_baseline / reference arm)
def oracle_sample(P, sample_bp):
    import oracle
    threads = len(os.sched_getaffinity(0))
    q_end = min(len(P.Q), sample_bp)
    t = time.perf_counter()
    out = oracle.mems(P.R, P.Q, P.L, P.ls, 0, 0, q_end, threads=threads)
    dt = time.perf_counter() - t
    oracle_sample.last = out
    return dt, q_end, len(out), oracle.num_threads(threads)


def run_reference(args, P):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    sample = min(len(P.Q), ORACLE_SAMPLE_BP["reference"])
    times = []
    for i in range(args.warmup + args.steps):
        dt, q_end, nm, cores = oracle_sample(P, sample)
        if i >= args.warmup:
            times.append(dt)
    t = statistics.mean(times)
    v = q_end / 1e6 / t
    desc = (f"full hash index of R ({len(P.R)} bp) + lookup/extension/sort-unique of MEMs starting in "
            f"Q[0:{q_end}] ({q_end / len(P.Q):.1%} of Q)")
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 3), "unit": "Mbp/s",
            "n_gpus": int(os.environ.get("WORLD_SIZE", "1")),
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8 (ASCII chars)",
            "data": "synthetic", "config": {"workload": WORKLOAD_DESC[args.config], "sample": desc},
            "cpu_baseline": {"value": round(v, 3), "unit": "Mbp/s", "cores": cores, "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": round(v, 3), "unit": "Mbp/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ roofline bookkeeping
def radix_passes(key_bits, n):
    """LSD passes the library's radix sort runs (radix.cu pick_digit_bits): 8-bit digits
    above 16 M keys, else 9-bit digits when that saves a pass, else 8-bit."""
    if n > (16 << 20):
        return (key_bits + 7) // 8
    return min((key_bits + 8) // 9, (key_bits + 7) // 8)


def d7_bytes(nR, nQ, ls, L, stats, mean_len):
    """SURVEY.md §8(d) D7's algorithmic bytes per step of each stage (what the method
    itself must move): pack 1.25 B per base; find per query position 0.25 B (packed Q)
    + 8 B (ptrs[s], ptrs[s+1]), per hit 4 B (locs) + 16 B (R window), per MEM
    mean_len/2 B (extension, R + Q) + 12 B (output); sort 12 B x 2 x passes per MEM."""
    pos, hits, mems = stats["positions"], stats["hits"], stats["mems"]
    kb = (max(nR, 1) - 1).bit_length() + (max(nQ, 1) - 1).bit_length()
    return {"pack": 1.25 * (nR + nQ),
            "find": (0.25 + 8) * pos + 20 * hits + (mean_len / 2 + 12) * mems,
            "sort": 24 * radix_passes(kb, mems) * mems}


def impl_bytes(nR, nQ, ls, L, stats):
    """Bytes this implementation's data structures must move per step,
    stage by stage; the find row is narrower than D7's (an occupancy bit and an 8-byte
    {first, count} entry per occupied seed instead of two ptrs reads per position; one
    seed record per hit instead of locs + an R window)."""
    step = L - ls + 1
    n_locs = (nR - ls) // step + 1 if nR >= ls else 0
    nb = 1 << (2 * ls)
    passes = radix_passes(2 * ls, n_locs)
    rec = 8 if step <= 8 else 16              # seed record bytes (index.cu)
    pos, occ, hits, mems = stats["positions"], stats["occupied"], stats["hits"], stats["mems"]
    sect = n_locs * 8 > (126 << 20) // 4      # rank sectors (16 B / 32 seeds) vs rank words (8 B)
    cap = pos // 8 + 4096                     # output capacity the pipeline sizes its sort for
    kb = (max(nR, 1) - 1).bit_length() + (max(nQ, 1) - 1).bit_length()
    sort = (mems * 56 if mems <= (2 << 20)    # MSD: histogram 8, scatter 24, local sort + triples 24
            else radix_passes(kb, cap) * mems * 32 + mems * 24)  # LSD: (8 + 4) x 2 + 8 per pass + triples
    return {
        "pack": 1.25 * (nR + nQ),
        "index.codes": n_locs * (8 + 8),
        "index.sort": passes * n_locs * (16 + 4),
        "index.ptrs": n_locs * 4 + (nb / 2 if sect else nb / 4) + 8 * min(n_locs, nb),
        "index.recs": n_locs * (4 + 24 + rec),
        # tiled Alg. 1 (tindex.cu, sparse indexes up to 2^20 locations): codes + locations
        # written, radix passes over the top 2 ls - 10 bits, the bins read once, locs +
        # {first, count} entry per location, the directory, the seed records
        "index.tiled": n_locs * (8 + radix_passes(max(2 * ls - 10, 0), n_locs) * 20 + 8 + 4 + 8 + 4 + 24 + rec)
                       + (nb / 2 if sect else nb / 4),
        "find": 0.25 * pos + pos / 8 + 8 * occ + rec * hits + 12 * mems,
        "sort": sort,
    }


# ------------------------------------------------------------------ D9 generator diagnostics
def d9_diagnostics(P, dev):
    """input SHA-256s, the Fig. 6 analogue (how many
    seeds have k = 1, 2, 3, ... sampled locations, and the largest bucket) and the
    distribution of hits per query position -- from the library's own index (the
    paper's dense ptrs, expanded on demand), outside the timed region."""
    import torch
    from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm
    shaR, shaQ = P.sha256()
    Rs = gm.pack(torch.from_numpy(P.R).to(dev))
    idx = gm.index_build(Rs, P.ls, P.L)
    ptrs, locs = idx.view()
    n_locs = locs.numel()
    cnt = (ptrs[1:].to(torch.int64) - ptrs[:-1].to(torch.int64))
    edges = [1, 2, 3, 4, 5, 8, 16, 32, 64, 128, 256, 1024, 4096]
    occupied = cnt[cnt > 0]
    fig6 = {"seeds_with_k_locs": {}, "occupied_seeds": int(occupied.numel()),
            "largest_bucket": int(occupied.max().item()) if occupied.numel() else 0}
    for a, b in zip(edges, edges[1:] + [None]):
        m = (occupied >= a) if b is None else ((occupied >= a) & (occupied < b))
        fig6["seeds_with_k_locs"][f"{a}+" if b is None else (str(a) if b == a + 1 else f"{a}-{b - 1}")] = \
            int(m.sum().item())
    # hits per query position = the bucket size of the position's seed (first base most significant)
    q = torch.from_numpy(P.Q).to(dev)
    c = ((q >> 1) ^ (q >> 2)) & 3  # A0 C1 G2 T3 (both cases)
    n = q.numel() - P.ls + 1
    hist = {}
    if n > 0:
        code = torch.zeros(n, dtype=torch.int64, device=dev)
        for i in range(P.ls):
            code = (code << 2) | c[i:i + n].to(torch.int64)
        h = cnt[code]
        for a, b in ((0, 1), (1, 2), (2, 4), (4, 16), (16, 64), (64, 256), (256, 1024), (1024, None)):
            m = (h >= a) if b is None else ((h >= a) & (h < b))
            hist[f"{a}+" if b is None else (str(a) if b == a + 1 else f"{a}-{b - 1}")] = int(m.sum().item())
        hist["mean"] = round(float(h.double().mean().item()), 4)
        hist["max"] = int(h.max().item())
        del code, h
    del cnt, occupied, ptrs, locs
    idx.free()
    Rs.free()
    return {"sha256_R": shaR, "sha256_Q": shaQ, "n_locs": int(n_locs), "fig6_bucket_sizes": fig6,
            "hits_per_position": hist}


# ------------------------------------------------------------------ our arm
def run_ours(args, P):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_abu_dolehkac14_b200 import gpumem as gm
    from paper_conf_ipps_abu_dolehkac14_b200.dist import ShardedPipeline

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # NCCL, one rank per GPU. GM_BENCH_BACKEND=gloo with GM_BENCH_SAME_DEVICE=1 runs the
    # N > 1 code path with every rank on cuda:0 (tests/test_gpu_bench.py: one GPU box)
    backend = os.environ.get("GM_BENCH_BACKEND", "nccl")
    gpu = 0 if os.environ.get("GM_BENCH_SAME_DEVICE") == "1" else local
    torch.cuda.set_device(gpu)
    if world > 1:
        dist.init_process_group(backend, device_id=torch.device("cuda", gpu) if backend == "nccl" else None)
    dev = torch.device("cuda", gpu)
    red_dev = dev if backend == "nccl" else torch.device("cpu")  # where the max-over-ranks reductions run
    stream = torch.cuda.current_stream()

    # inputs resident in HBM before timing
    R_dev = torch.from_numpy(P.R).to(dev)
    Q_dev = torch.from_numpy(P.Q).to(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    torch.cuda.synchronize()

    # the step: one CUDA-graph launch of the whole path per rank (pack R, pack Q, index,
    # find over the rank's shard, output sort); for N > 1 also the gather + rank-0 merge
    # (captured with event nodes around the find kernel only: every stage boundary as an
    # event-record node would add ~50 us per step; the full breakdown is a separate run)
    gm.set_option("pipe_events", 2)
    sp = ShardedPipeline(len(P.R), len(P.Q), P.L, P.ls)
    n_mems, stats = 0, None
    for _ in range(args.warmup):
        flush.zero_()
        sp.run(R_dev, Q_dev)
        n_mems = sp.finish() or 0
        stats = sp.pl.stats()
    torch.cuda.synchronize()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    prof = {}
    fallbacks = 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = gm.launch_count()
    host_ms = []
    with ClockSampler(gpu) as clk:
        for i in range(args.steps):
            flush.zero_()
            ev[i][0].record(stream)
            th = time.perf_counter()
            sp.run(R_dev, Q_dev)
            if world > 1:  # the exchange needs the counts: result, gather, merge inside the step
                sp.finish()
                ev[i][1].record(stream)
            else:
                ev[i][1].record(stream)
                sp.finish()  # sync + capacity check outside the step's events
                if sp.pl.stats()["attempts"] > 1:  # overflow rerun ran after ev[i][1]: time it too
                    fallbacks += 1
                    ev[i] = (ev[i][0], torch.cuda.Event(enable_timing=True))
                    ev[i][1].record(stream)
            host_ms.append(1e3 * (time.perf_counter() - th))
            for k, (t, nl) in sp.pl.profile().items():  # find's event nodes inside this launch
                a0 = prof.get(k, (0.0, 0))
                prof[k] = (a0[0] + t, a0[1] + nl)
        torch.cuda.synchronize()
    launches = gm.launch_count() - l0
    # the last timed step's MEMs (rank 0's merged set for N > 1)
    gpu_result = sp.pl.numpy() if world == 1 else (sp.merged.numpy() if rank == 0 else None)
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    tot = torch.tensor([sum(step_ms)], dtype=torch.float64, device=red_dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    ms = tot.item() / args.steps
    value = len(P.Q) / 1e6 / (ms / 1e3)

    # ---- per-stage breakdown: a separate short run of a pipeline captured with an event
    # node at every stage boundary (outside the timed region; those nodes cost ~50 us)
    gm.set_option("pipe_events", 1)
    spp = ShardedPipeline(len(P.R), len(P.Q), P.L, P.ls) if world == 1 else None
    stage_prof, n_prof = {}, 5
    if spp is not None:
        for i in range(2 + n_prof):
            flush.zero_()
            spp.run(R_dev, Q_dev)
            spp.finish()
            if i >= 2:
                for k, (t, nl) in spp.pl.profile().items():
                    a0 = stage_prof.get(k, (0.0, 0))
                    stage_prof[k] = (a0[0] + t, a0[1] + nl)
        spp.free()
    gm.set_option("pipe_events", 0)
    stage_ms_all = {k: v[0] / n_prof for k, v in stage_prof.items()}

    # ---- roofline of the dominant kernel (k_find: the largest share of the step), its
    # time measured live in the timed region by the graph's event nodes around it
    kernel_ms = {k: v[0] / args.steps for k, v in prof.items()}
    dom = max(kernel_ms, key=kernel_ms.get)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = peaks.get("hbm_gbs", 6650.0)
    peak_src = "measured" if "hbm_gbs" in peaks else "fallback"
    nQ, nR, ls, L = len(P.Q), len(P.R), P.ls, P.L
    step_ = L - ls + 1
    mean_len = float(gpu_result[:, 2].astype(np.float64).mean()) if gpu_result is not None and len(gpu_result) else \
        float(L)
    d7 = d7_bytes(nR, nQ, ls, L, stats, mean_len)
    alg = impl_bytes(nR, nQ, ls, L, stats)
    roof = None
    if dom in d7:
        n_launch = prof[dom][1] / args.steps
        sec = kernel_ms[dom] / 1e3
        achieved = d7[dom] / sec / 1e9
        achieved_impl = alg[dom] / sec / 1e9
        traffic, sectors = None, None
        try:  # dram read+write bytes of that kernel from the committed ncu --set full capture
            t = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json"))).get(args.config)
            if t and dom == "find" and world == 1:
                traffic = int(t["traffic_bytes"])
                sectors = t.get("l1_ld_sectors")
        except Exception:
            pass
        roof = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": peak,
                "peak_source": peak_src, "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                "bytes_model": "SURVEY.md §8(d) D7: 8.25 B per query position + 20 B per hit + "
                               "(mean_len/2 + 12) B per MEM",
                "algorithmic_bytes_per_step": int(d7[dom]), "mean_mem_len": round(mean_len, 2),
                "frac_d7": round(achieved / peak, 4),
                "impl_bytes_per_step": int(alg[dom]), "achieved_impl": round(achieved_impl, 1),
                "frac_impl": round(achieved_impl / peak, 4),
                "impl_bytes_model": "DESIGN.md §7: this build's structures (occupancy bit per position, "
                                    "8 B entry per occupied seed, one seed record per hit, 12 B per MEM)",
                "launches_per_step": n_launch, "ms_per_step": round(kernel_ms[dom], 4)}
        if traffic:
            roof["traffic_over_d7"] = round(traffic / d7[dom], 3)
        if sectors:  # what bounds k_find: 32-byte sector requests L1 -> L2, ceiling
            # ~1 sector per SM clock; ncu's sector count over the live kernel time and SM clock
            clk_mhz = (clk.summary().get("sm_mhz") or 1965.0)
            rate = sectors / (torch.cuda.get_device_properties(dev).multi_processor_count * clk_mhz * 1e6
                              * kernel_ms[dom] / 1e3 / n_launch)
            roof["l1_sectors_per_launch"] = int(sectors)
            roof["l1_sector_rate_per_sm_clk"] = round(rate, 3)
            # the same number of random 8-byte probes into an L2-resident table the size of
            # the rank directory, nothing else (gpumem_gather_ceiling), measured here: the
            # practical peak of k_find's access pattern on this GPU
            try:
                table = (1 << (2 * ls)) // 32 * 16  # the directory: 16 B per group of 32 seeds
                ceil_ms = gm.gather_ceiling(int(sectors), table)
                find_ms = kernel_ms[dom] / n_launch
                dram_gbs = traffic / (find_ms / 1e3) / 1e9 if traffic else 0.0
                roof["note"] = ("k_find is DRAM-bound here (random seed-record gathers at 64-B DRAM granularity)"
                                if dram_gbs > 0.4 * peak else
                                "k_find is bound by random L1->L2 requests and their latency chain (directory "
                                "probe -> bucket entry -> seed record), not HBM bandwidth (DESIGN.md §7)")
                roof["gather_ceiling"] = {
                    "what": f"{int(sectors)} random 8-B loads into a {table >> 20} MB table, 8 per thread",
                    "unit": "Gsector/s", "peak": round(sectors / ceil_ms / 1e6, 1),
                    "achieved": round(sectors / find_ms / 1e6, 1), "frac": round(ceil_ms / find_ms, 3)}
            except Exception as e:  # pragma: no cover
                roof["gather_ceiling"] = {"error": repr(e)}
    stage_frac = {k: round(alg[k] / (stage_ms_all[k] / 1e3) / 1e9 / peak, 4) for k in alg if k in stage_ms_all}
    stage_frac_d7 = {k: round(d7[k] / (stage_ms_all[k] / 1e3) / 1e9 / peak, 4) for k in d7 if k in stage_ms_all}

    line = {"metric": METRIC, "value": round(value, 2), "unit": "Mbp/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u64 (2-bit packed bases), u32 positions", "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC[args.config], "R_bp": nR, "Q_bp": nQ, "L": L, "ls": ls,
                       "step": step_, "mems": n_mems, "l2": "flushed before every step (512 MB write)",
                       "parallelism": f"query-sharded dp{world}, index rebuilt per rank, NCCL gather + merge",
                       "inputs": "ASCII R, Q resident in HBM at t0"},
            "mems_per_s": round(n_mems / (ms / 1e3), 1),
            "stage_ms": {k: round(v, 4) for k, v in sorted(stage_ms_all.items())},
            "stage_ms_note": "separate 5-step run with an event node at every stage boundary (not the timed region)",
            "find_ms_live": round(kernel_ms.get("find", 0.0), 4),
            "stage_hbm_frac": stage_frac, "stage_hbm_frac_d7": stage_frac_d7, "find_stats": stats,
            "work_balance": {  # the tile scheduler's balance
                "what": "hits dealt by the busiest warp of k_find vs the mean over its warps (heavy-queue hits, "
                        "drained by k_heavy, are not a warp's own)",
                "max_warp_hits": stats.get("max_warp_hits"), "warps": stats.get("warps"),
                "max_over_mean": round(stats["max_warp_hits"] * stats["warps"] / max(1, stats["hits"]), 3)
                if stats.get("warps") else None},
            "gpu_launches": int(launches),
            "clocks": clk.summary(), "roofline": roof,
            "host_ms_per_step": round(statistics.mean(host_ms), 4), "capacity_fallbacks": fallbacks,
            "launch_mode": "one CUDA graph per step (gpumem_pipeline_run)",
            "step_ms_minmax": [round(min(step_ms), 4), round(max(step_ms), 4)]}

    # ---- end-to-end through the public API with HOST buffers (pinned), H2D + D2H inside:
    # gpumem_pipeline_run_host copies R then Q on a copy stream while the graph packs and
    # indexes R; then the sorted triples come back to pinned host memory
    if not args.no_e2e and world == 1:
        R_h = torch.from_numpy(P.R).pin_memory()
        Q_h = torch.from_numpy(P.Q).pin_memory()
        pe = gm.Pipeline(nR, nQ, ls, L)
        host_out = None
        times = []
        nm = 0
        for i in range(args.e2e_steps + 2):
            flush.zero_()
            torch.cuda.synchronize()
            t = time.perf_counter()
            pe.run_host(R_h, Q_h)
            nm = pe.result()
            if host_out is None or host_out.shape[0] < nm:
                host_out = torch.empty((max(nm, 1) * 5 // 4, 3), dtype=torch.uint32, pin_memory=True)
            if nm:
                host_out[:nm].copy_(pe.view_u32(), non_blocking=True)
            torch.cuda.current_stream().synchronize()
            dt = time.perf_counter() - t
            if i >= 2:  # the first run captures the graph, the second allocates the pinned output
                times.append(dt)
        pe.free()
        te = statistics.median(times)  # host wall clock: the median resists a stray OS hiccup
        line["e2e"] = {"value": round(nQ / 1e6 / te, 2), "unit": "Mbp/s", "h2d_bytes_per_step": nR + nQ,
                       "d2h_bytes_per_step": 12 * nm + 128, "ms_per_step": round(te * 1e3, 3),
                       "ms_minmax": [round(min(times) * 1e3, 3), round(max(times) * 1e3, 3)],
                       "steps": args.e2e_steps,
                       "path": "gpumem_pipeline_run_host (pinned host R, Q) + result + D2H of the triples"}

    if not args.no_e2e and world > 1:
        # every rank: its shard's pipeline from pinned host R and Q (the whole of both: a
        # shard's extensions read all of Q), the fused gather + merge, and on rank 0 the
        # D2H of the merged triples; the max over ranks of the median wall time
        R_h = torch.from_numpy(P.R).pin_memory()
        Q_h = torch.from_numpy(P.Q).pin_memory()
        se = ShardedPipeline(nR, nQ, L, ls)
        host_out, times, nm = None, [], 0
        for i in range(args.e2e_steps + 2):
            flush.zero_()
            torch.cuda.synchronize()
            dist.barrier()
            t = time.perf_counter()
            se.run_host(R_h, Q_h)
            nm = se.finish() or 0
            if rank == 0:
                if host_out is None or host_out.shape[0] < nm:
                    host_out = torch.empty((max(nm, 1) * 5 // 4, 3), dtype=torch.uint32, pin_memory=True)
                if nm:
                    host_out[:nm].copy_(se.merged.view_u32(), non_blocking=True)
            torch.cuda.current_stream().synchronize()
            if i >= 2:
                times.append(time.perf_counter() - t)
        te_t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=red_dev)
        dist.all_reduce(te_t, op=dist.ReduceOp.MAX)
        te = te_t.item()
        se.free()
        line["e2e"] = {"value": round(nQ / 1e6 / te, 2), "unit": "Mbp/s", "h2d_bytes_per_step": world * (nR + nQ),
                       "d2h_bytes_per_step": 12 * nm + 128 * world, "ms_per_step": round(te * 1e3, 3),
                       "steps": args.e2e_steps,
                       "path": "per rank: gpumem_pipeline_run_host (pinned host R, Q) of its shard; fused gather + "
                               "merge on rank 0 (dist.ShardedPipeline); D2H of the merged triples on rank 0; "
                               "max over ranks"}

    # ---- D9 generator diagnostics (input digests, Fig. 6 bucket sizes, hits per position)
    if rank == 0 and not args.no_d9:
        try:
            line["d9"] = d9_diagnostics(P, dev)
        except Exception as e:  # pragma: no cover
            line["d9"] = {"error": repr(e)}

    # ---- CPU oracle on a bounded sample (rank 0, N = 1 only)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        dt, q_end, nm_cpu, cores = oracle_sample(P, ORACLE_SAMPLE_BP["ours"])
        line["cpu_baseline"] = {
            "value": round(q_end / 1e6 / dt, 3), "unit": "Mbp/s", "cores": cores, "kind": "oracle",
            "sample": f"full hash index of R + MEMs starting in Q[0:{q_end}] ({q_end / nQ:.1%} of Q); "
                      f"{nm_cpu} MEMs in {dt:.2f} s"}
        # parity on the same sample: the timed pipeline's last result restricted to MEM
        # starts q < q_end (sorted by (r, q), so the restriction keeps the order) against
        # the oracle's triples, element by element
        import hashlib
        want = np.ascontiguousarray(oracle_sample.last, dtype=np.uint32)
        got = gpu_result[gpu_result[:, 1] < q_end] if gpu_result is not None else np.zeros((0, 3), np.uint32)
        got = np.ascontiguousarray(got, dtype=np.uint32)
        line["parity_sample"] = {"q_range": [0, int(q_end)], "mems_gpu": int(len(got)), "mems_oracle": int(len(want)),
                                 "equal": bool(got.shape == want.shape and np.array_equal(got, want)),
                                 "sha256_gpu": hashlib.sha256(got.tobytes()).hexdigest()[:16],
                                 "sha256_oracle": hashlib.sha256(want.tobytes()).hexdigest()[:16]}
    if world > 1:
        dist.barrier()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def relaunch_under_torchrun(args):
    """`bench.py --gpus N` (N > 1) outside a launcher: run the same command as N ranks,
    one per GPU, under torch.distributed.run (the driver's own launch), and exit with
    its status."""
    import socket
    import subprocess
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    sys.exit(subprocess.call(cmd))


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "0"))
    if world == 0 and args.gpus > 1:
        relaunch_under_torchrun(args)
    if world and world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} ranks were launched")
    P = synth.make_pair(args.config)
    if args.impl == "reference":
        run_reference(args, P)
    else:
        run_ours(args, P)


if __name__ == "__main__":
    main()
