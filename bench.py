#!/usr/bin/env python
"""Benchmark of the FastZ hot path on B200 (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl fastz|reference]

Headline workload (BASELINE.json configs[2], "C3", the largest single-GPU config): synthetic 100 Mbp
chromosome-scale pair, 2^21 seeds per GPU, with 16-64 kbp high-scoring alignments among the paper's skewed
length mix (synth.genome.config3).  One step = one fastz_extend_seeds call over the
whole seed batch: inspector + eager traceback, binning, trimmed executor, traceback and CIGAR assembly, seeds
and sequences resident in HBM (``value``); ``e2e`` repeats it through the public API from pinned host seeds to
host records + CIGAR text.  ``secondary`` holds the same measurement on C2 (10 Mbp, 2^20 seeds).

``genome_pair`` (whole-genome-pair wall time on C4, 2^30 bp x 2^30 bp, 2^23 seeds): the
multi-GPU driver ``dist.extend_genome_pair`` over all N ranks -- rank 0 packs and broadcasts the sequences
(2 bits per base) and the seeds, every rank extends its hash shard, records are gathered to rank 0 over NCCL and
put back in seed order, results end on rank 0's host; max over ranks of the device-synchronised wall clock.

Metric: GCUPS = explored DP cells (origin + cells with a live neighbour, reading R7 -- the exact
count, produced once by the census kernel and parity-tested against the oracle) / step time.  Multi-GPU:
each rank extends its own 2^21-seed shard of the same pair, nothing is exchanged in the timed region (scaling
"weak"); time = max over ranks.

--impl reference times the CPU oracle (oracle/, the plain sequential implementation) on a bounded sample
of the same workload on this box's host cores; it is the reference arm of this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# algorithmic integer ops per explored cell: the recurrences' 4 max + 5 add.
# The cone y-drop adds 4 more (2 max, 1 add, 1 compare), reported separately as frac_with_ydrop.
OPS_PER_CELL = 9
OPS_PER_CELL_YDROP = 13
PAPER_CONTEXT = {"fastz_rtx3080_vs_sequential_lastz": 111, "multicore_lastz_16c_vs_sequential": 20,
                 "source": "PAPER.md P:22, P:279-281 (context only: different baseline program and hardware)"}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--seeds", type=int, default=0, help="seeds per GPU (default: the config's)")
    ap.add_argument("--impl", default="fastz", choices=["fastz", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-secondary", action="store_true", help="skip the C2 secondary measurement")
    ap.add_argument("--no-genome-pair", action="store_true", help="skip the C4 genome-pair wall time")
    ap.add_argument("--profile", action="store_true", help="one warm-up + 1 step of the headline only, for ncu")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


DESC = {
    1: "C1: synthetic 100 kbp target vs mutated copy (~10% subs, 1% indels), 2,048 seeds",
    2: "C2: synthetic 10 Mbp chromosome pair, 2^20 seeds per GPU, skewed extension lengths (>97% <=128 bp)",
    3: "C3: synthetic 100 Mbp chromosome-scale pair, 2^21 seeds per GPU, long (16-64 kbp) high-scoring alignments",
    5: "C5: extension-length stress sweep 32 bp - 64 kbp, 2^20 seeds per GPU",
    6: "C6 (NEXT-2): dissimilar 10 Mbp pair, diverged short homology (cross-genus analog, P:331-340)",
}
DEFAULT_SEEDS = {1: 2048, 2: 1 << 20, 3: 1 << 21, 5: 1 << 20, 6: 1 << 20}


def workload(config: int, n_per_gpu: int, world: int, rank: int):
    from synth import genome
    if config not in DESC:
        raise SystemExit(f"config {config} not supported by bench")
    n = n_per_gpu or DEFAULT_SEEDS[config]
    w = genome.make(config, n_seeds=n * world)
    shard = w.seeds[rank::world][:n]
    return w, shard, DESC[config]


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={gpu}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-lms", "200"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = [r.split(",") for r in open(self.f.name).read().strip().splitlines() if r.strip()]
        os.unlink(self.f.name)
        sm = [float(r[1]) for r in rows if len(r) > 8 and r[1].strip().replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) > 8 and r[2].strip().replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            if len(r) > 8:
                for k, nm in enumerate(names):
                    if "Active" in r[5 + k] and "Not" not in r[5 + k]:
                        reasons.add(nm)
        loaded = [s for s in sm if s > 500] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


def host_cpu():
    """CPU model, clock and usable cores of this host (lscpu / /proc/cpuinfo)."""
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()
    model, mhz = None, None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() == "Model name":
                model = v.strip()
            elif k.strip() in ("CPU max MHz", "CPU MHz") and mhz is None:
                mhz = float(v.strip())
    except Exception:
        pass
    if mhz is None:
        try:
            for line in open("/proc/cpuinfo"):
                if line.startswith("cpu MHz"):
                    mhz = float(line.split(":")[1])
                    break
        except Exception:
            pass
    return {"model": model, "mhz": mhz, "cores": cores}


def _oracle_rate(w, seeds, threads, target_s, rng):
    """Oracle cells/s on a random sample of ``seeds`` sized for about ``target_s`` seconds."""
    from oracle import core
    n = min(len(seeds), max(16, 4 * threads))
    for _ in range(4):
        idx = rng.choice(len(seeds), n, replace=False)
        t0 = time.perf_counter()
        r = core.extend(w.T, w.Q, seeds[idx], threads=threads)
        dt = time.perf_counter() - t0
        if dt >= target_s / 3 or n >= len(seeds):
            break
        n = min(len(seeds), int(n * target_s / max(dt, 1e-3)))
    cells = int(r.rec["l_explored"].sum() + r.rec["r_explored"].sum())
    return cells / dt, n, cells, dt


def cpu_baseline(w, seeds, gpu_gcups):
    """The oracle as it stands on this box's host cores (all of them, and one), on bounded random samples of
    the same workload; GPU speed-ups beside the paper's (context)."""
    import numpy as np
    cpu = host_cpu()
    rng = np.random.default_rng(12345)
    rate_all, n_all, cells_all, dt_all = _oracle_rate(w, seeds, cpu["cores"], 15.0, rng)
    rate_1, n_1, cells_1, dt_1 = _oracle_rate(w, seeds, 1, 6.0, rng)
    return {"value": rate_all / 1e9, "unit": "GCUPS", "cores": cpu["cores"], "kind": "oracle",
            "sample": f"{n_all} random seeds of the same workload ({cells_all} explored cells) in {dt_all:.2f} s on "
                      f"{cpu['cores']} threads; 1-thread rate from {n_1} seeds ({cells_1} cells) in {dt_1:.2f} s",
            "cpu_model": cpu["model"], "cpu_mhz": cpu["mhz"],
            "one_core_gcups": rate_1 / 1e9, "seeds_per_s": n_all / dt_all,
            "gpu_speedup_vs_all_cores": gpu_gcups / (rate_all / 1e9),
            "gpu_speedup_vs_one_core": gpu_gcups / (rate_1 / 1e9),
            "paper_context": PAPER_CONTEXT}


def run_reference(args, ws, rank):
    if rank != 0:
        return
    import numpy as np
    from oracle import core
    w, seeds, desc = workload(args.config, args.seeds, 1, 0)
    cpu = host_cpu()
    cores = cpu["cores"]
    rng = np.random.default_rng(777)
    per = max(64, 6 * cores)
    # calibrate so one step takes ~8 s on this host
    t0 = time.perf_counter()
    core.extend(w.T, w.Q, seeds[rng.choice(len(seeds), per, replace=False)], threads=cores)
    dt = time.perf_counter() - t0
    per = int(min(len(seeds), max(per, per * 8.0 / max(dt, 1e-3))))
    for _ in range(args.warmup):
        core.extend(w.T, w.Q, seeds[rng.choice(len(seeds), min(per, 64), replace=False)], threads=cores)
    tot_cells, tot_t = 0, 0.0
    for _ in range(args.steps):
        idx = rng.choice(len(seeds), per, replace=False)
        t0 = time.perf_counter()
        r = core.extend(w.T, w.Q, seeds[idx], threads=cores)
        tot_t += time.perf_counter() - t0
        tot_cells += int(r.rec["l_explored"].sum() + r.rec["r_explored"].sum())
    v = tot_cells / tot_t / 1e9
    line = {"impl": "reference", "metric": "GCUPS", "value": v, "unit": "GCUPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": tot_t / args.steps * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "config": {"workload": desc, "seeds_per_step": per, "sample": "random seeds of the workload per step"},
            "cpu_baseline": {"value": v, "unit": "GCUPS", "cores": cores, "kind": "oracle",
                             "cpu_model": cpu["model"], "cpu_mhz": cpu["mhz"],
                             "sample": f"{per} random seeds per step x {args.steps} steps"},
            "e2e": {"value": v, "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def measure(al, seeds_d, steps, warmup, stream, flush, ws, clocks=None):
    """Device-timed steps (CUDA events on the library's stream, L2 flushed between steps, untimed)."""
    import torch
    import torch.distributed as dist
    for _ in range(warmup):
        al.extend_only(seeds_d)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    clk = clocks() if clocks else None
    times, stages, launches = [], [], 0
    for _ in range(steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        al.extend_only(seeds_d)
        e1.record(stream)
        e1.synchronize()
        times.append(e0.elapsed_time(e1))
        s = al.stats()
        stages.append(s)
        launches += int(s["n_launches"])
    torch.cuda.synchronize()
    clk_rec = clk.stop() if clk else None
    if ws > 1:
        dist.barrier()
    return times, stages, launches, clk_rec


def genome_pair(ws, rank, local):
    """C4 whole-genome-pair wall time through dist.extend_genome_pair on all ranks (rank 0's host ASCII + seeds
    -> rank 0's host records + CIGARs); first (cold: context + pool allocation) and second (warm) run."""
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sc_gundaboluvt21_b200 import dist as fzdist
    w = None
    t_gen = 0.0
    if rank == 0:
        from synth import genome
        t0 = time.perf_counter()
        w = genome.config4()
        t_gen = time.perf_counter() - t0
    runs = []
    for _ in range(2):
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        tm = {}
        t0 = time.perf_counter()
        rec, cig = fzdist.extend_genome_pair(w.T if w else None, w.Q if w else None, w.seeds if w else None,
                                             timings=tm, torch_alloc=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        t = torch.tensor([dt, tm["broadcast_s"], tm["extend_s"], tm["gather_s"]], dtype=torch.float64,
                         device=torch.device("cuda", local))
        if ws > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        runs.append([float(x) for x in t.tolist()])
        if rank == 0:
            n = len(rec)
            cbytes = len(cig)
        del rec, cig
    if rank != 0:
        return None
    cold, warm = runs
    return {"workload": "C4: synthetic 2^30 bp x 2^30 bp genome pair, 2^23 seeds (C2 block mix x100), LASTZ default "
                        "scoring", "n_gpus": ws, "seeds": n, "cigar_bytes": cbytes,
            "wall_s": warm[0], "cold_wall_s": cold[0],
            "phases_s_max_over_ranks": {"broadcast": warm[1], "extend": warm[2], "gather_merge_d2h": warm[3]},
            "seed_extensions_per_s": n / warm[0],
            "timing": "time.perf_counter around extend_genome_pair after a barrier and device sync, max over ranks; "
                      "2-bit sequence broadcast, extension, NCCL gather + seed-order merge, copy to rank 0's host "
                      "included; seed finding and input generation excluded",
            "generation_s": t_gen}


def run_fastz(args, ws, rank, local):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sc_gundaboluvt21_b200 import fastz

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)
    w, shard, desc = workload(args.config, args.seeds, ws, rank)
    n = len(shard)
    al = fastz.Aligner(w.T, w.Q, device=local, stream=stream.cuda_stream, torch_alloc=True)
    seeds_d = torch.from_numpy(np.ascontiguousarray(shard)).to(dev)
    seeds_h = torch.from_numpy(np.ascontiguousarray(shard)).pin_memory()

    # exact explored-cell count (GCUPS numerator), untimed
    al.extend_only(seeds_d)
    cells = int(al.census().sum())
    st0 = al.stats()
    peak_ops, peak_mhz = fastz.fastz_int_peak(local, 300.0)

    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    if args.profile:
        args.warmup, args.steps = 1, 1
    times, stages, launches, clocks = measure(al, seeds_d, args.steps, args.warmup, stream, flush, ws,
                                              clocks=lambda: Clocks(local))
    ms = sum(times) / len(times)
    if args.profile:
        al.close()
        if rank == 0:
            print(json.dumps({"profile": True, "ms_per_step": ms}), flush=True)
        return

    # e2e through the public API: pinned host seeds -> host records + CIGAR (the Aligner's page-locked result
    # buffers are allocated once, untimed, as a long-running user would keep them)
    al.results_pinned()
    e2e_t = []
    d2h = 0
    for _ in range(max(1, min(args.steps, 3))):
        flush.zero_()
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        t0 = time.perf_counter()
        al.extend_only(seeds_h)
        res = al.results_pinned()
        e2e_t.append(time.perf_counter() - t0)
        d2h = res.rec.nbytes + len(res.cigar)
    e2e_ms = sum(e2e_t) / len(e2e_t) * 1e3
    al.close()

    # secondary: the same device-timed step on C2 (10 Mbp pair, 2^20 seeds per GPU), plus the NEXT-4 seeding
    # and NEXT-3 post-pass stages on that pair (rank 0)
    secondary, seeding, dedup = None, None, None
    if not args.no_secondary:
        w2, shard2, desc2 = workload(2, 0, ws, rank)
        al2 = fastz.Aligner(w2.T, w2.Q, device=local, stream=stream.cuda_stream, torch_alloc=True)
        s2 = torch.from_numpy(np.ascontiguousarray(shard2)).to(dev)
        al2.extend_only(s2)
        cells2 = int(al2.census().sum())
        t2, st2, _l2, _c = measure(al2, s2, 3, 3, stream, flush, ws)
        ms2 = sum(t2) / len(t2)
        secondary = {"workload": desc2, "value": cells2 / (ms2 * 1e-3) / 1e9, "unit": "GCUPS", "ms_per_step": ms2,
                     "inspector_ms": sum(s["ms_inspect"] for s in st2) / len(st2), "cells_per_gpu": cells2,
                     "roofline_frac": OPS_PER_CELL * cells2 / (sum(s["ms_inspect"] for s in st2) / len(st2) * 1e-3)
                     / peak_ops}
        if rank == 0:
            try:
                al2.find_hsps()
                ts = []
                for _ in range(3):
                    torch.cuda.synchronize()
                    t1 = time.perf_counter()
                    hs, _an, hits = al2.find_hsps()
                    torch.cuda.synchronize()
                    ts.append(time.perf_counter() - t1)
                seeding = {"stage": "seeding + ungapped filter (fastz_find_hsps: 12of19 spaced seeds + transitions, "
                                    "x-drop 910, HSP >= 3000), C2 pair", "ms": min(ts) * 1e3, "hits": hits,
                           "hsps": int(len(hs)), "query_mbp_per_s": len(w2.Q) / min(ts) / 1e6}
            except Exception as e:  # reported, never fatal for the headline line
                seeding = {"error": str(e)[:200]}
            try:
                al2.extend_only(s2)
                al2.mark_redundant()
                ts = []
                for _ in range(3):
                    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    torch.cuda.synchronize()
                    ev0.record(stream)
                    _red, nred = al2.mark_redundant()
                    ev1.record(stream)
                    ev1.synchronize()
                    ts.append(ev0.elapsed_time(ev1))
                nk = int((al2.results().rec["flags"] & fastz.FLAG_ABOVE_K != 0).sum())
                dedup = {"stage": "redundant-alignment post-pass (fastz_mark_redundant, reading R14), C2 batch, "
                                  "incl. the D2H of the per-seed marks", "ms": min(ts), "above_k": nk,
                         "redundant": int(nred)}
            except Exception as e:
                dedup = {"error": str(e)[:200]}
        al2.close()
        del w2

    t = torch.tensor([ms, e2e_ms, float(cells), float(n)], dtype=torch.float64, device=dev)
    if ws > 1:
        tmax = t.clone()
        dist.all_reduce(tmax[:2], op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum[2:], op=dist.ReduceOp.SUM)
        ms, e2e_ms = float(tmax[0]), float(tmax[1])
        cells_all, n_all = float(tsum[2]), float(tsum[3])
    else:
        cells_all, n_all = float(cells), float(n)
    del al
    gp = None
    if not args.no_genome_pair:
        try:
            gp = genome_pair(ws, rank, local)
        except Exception as e:  # reported, never fatal for the headline line
            gp = {"error": str(e)[:300]} if rank == 0 else None
    if rank != 0:
        return
    value = cells_all / (ms * 1e-3) / 1e9
    insp_ms = sum(s["ms_inspect"] for s in stages) / len(stages)
    achieved = OPS_PER_CELL * cells / (insp_ms * 1e-3)
    traffic, traffic_src = None, None
    tf = os.path.join(ROOT, "profiles", "inspector_traffic.json")
    if os.path.exists(tf):
        try:
            tj = json.load(open(tf))
            entry = tj.get(f"C{args.config}")
            if entry:
                traffic = entry.get("bytes_per_launch")
                traffic_src = "constant from an ncu --set full capture, not measured in this run: " + entry.get("source", "")
        except Exception:
            traffic = None
    avg = lambda k: sum(s[k] for s in stages) / len(stages)  # noqa: E731
    line = {
        "metric": "GCUPS", "value": value, "unit": "GCUPS", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u16x2+int32",
        "data": "synthetic",
        "config": {"workload": desc, "seeds_per_gpu": n, "target_bp": len(w.T), "query_bp": len(w.Q),
                   "l2": "flushed between timed steps (256 MiB write, untimed)",
                   "rows_per_lane": int(os.environ.get("FASTZ_R", "4")), "parallelism": f"seed-sharded x{ws}"},
    }
    line.update({
        "seed_extensions_per_s": n_all / (ms * 1e-3),
        "cells": cells_all,
        "clocks": clocks,
        "e2e": {"value": cells_all / (e2e_ms * 1e-3) / 1e9, "unit": "GCUPS", "ms_per_step": e2e_ms,
                "h2d_bytes_per_step": int(n * 16), "d2h_bytes_per_step": int(d2h)},
        "gpu_launches": launches,
        "genome_pair": gp,
        "secondary": secondary,
        "seeding": seeding,
        "dedup": dedup,
        "roofline": {"bound": "alu", "kernel": ("inspector stage: k_inspect_mixed (packed u16x2, two sides per warp) + "
                                                "k_inspect (predicted-long sides, concurrent stream) + k_eager"
                                                if st0.get("n_packed_sides", 0) else "k_inspect"),
                     "achieved": achieved / 1e12, "peak": peak_ops / 1e12,
                     "unit": "Tops/s (INT32 lane ops)", "frac": achieved / peak_ops, "traffic": traffic,
                     "traffic_source": traffic_src, "ops_per_cell": OPS_PER_CELL,
                     "frac_with_ydrop": OPS_PER_CELL_YDROP * cells / (insp_ms * 1e-3) / peak_ops,
                     "inspector_ms": insp_ms, "inspector_share_of_step": insp_ms / ms,
                     "algorithmic": f"{OPS_PER_CELL} int ops per explored cell (P:63, P:346: 4 max + 5 add) x "
                                    f"{cells} explored cells per launch / mean inspector-stage time (CUDA events)",
                     "peak_source": f"measured fastz_int_peak (IMNMX/IADD3/VIADDMNMX chains on the ALU + FMA pipes, "
                                    f"128 lane-ops/clk/SM) at {peak_mhz:.0f} MHz; guide-derived 148 SMs x 4 SMSPs x "
                                    f"2 pipes x 16 lanes/clk x 1.965 GHz = 37.2 T/s"},
        "stages_ms": {k: avg(k) for k in ("ms_upload", "ms_inspect", "ms_bin", "ms_execute", "ms_traceback",
                                          "ms_combine")},
        "inspector_sides": {"packed": st0.get("n_packed_sides", 0), "long_32bit": st0.get("n_long_sides", 0),
                            "redone_32bit": st0.get("n_redo_sides", 0)},
        "bins_per_side": st0["bin_counts"][:7], "exec_sides": st0["n_exec_sides"], "eager_sides": st0["n_eager_sides"],
        "exec_words": st0["exec_words"], "exec_reserved_words": st0["exec_reserved_words"],
        "wide_sides": st0["n_wide_sides"], "executor_waves": st0["n_waves"],
    })
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(w, shard, value / ws)
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    ws, rank, local = dist_env()
    if ws > 1:
        import torch
        import torch.distributed as dist
        if args.impl == "reference":
            if rank != 0:
                return
            run_reference(args, ws, 0)
            return
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    if args.impl == "reference":
        run_reference(args, ws, rank)
        return
    run_fastz(args, ws, rank, local)
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
