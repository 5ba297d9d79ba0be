#!/usr/bin/env python
"""Benchmark of the B200 local-assembly hot path.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl ours|reference]

A step = one la_extend over the whole batch: plan, shared-memory-table kernel (build + ext rule +
walk + k retry for every small/medium end), global-memory rounds for the heavy ends, compaction.
`value` = extended bases/s with the inputs resident in HBM (device-timed with CUDA events on the
library's stream, max over ranks); `e2e` = the same metric through the public API from pinned host
buffers (H2D + encode + extend + D2H of all results inside the timed region).
N > 1 (torchrun, one process per GPU, NCCL): weak scaling — every rank extends its own shard of
the paper-shaped workload (an independent synthetic sample, seed + rank), no collective on the
data path, one result gather to rank 0 after the timed region.
The reference arm (--impl reference) is the CPU oracle (oracle/), timed on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "extended bases/s"
UNIT = "bases/s"
CONFIG_DESC = {
    "C1": "C1 tiny single-genome check (50 kbp, 200 contigs, 20k error-free reads, k=21)",
    "C2": "C2 synthetic 20-species metagenome (~37k contigs, 1% errors, full k 33/21/99/8 schedule)",
    "C3": "C3 high-skew (18 ends with >40k reads + ~60k sparse ends)",
    "C4": "C4 paper-shaped batch (500-species metagenome, lognormal(0,1.5), 150 bp pairs) on 1 B200",
}
CACHE = os.environ.get("LA_GEN_CACHE", "/tmp/la_gen_cache")


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def load_workload(config, seed, scale):
    """Deterministic synthetic batch; cached on local disk by (config, seed, scale) to save
    regeneration time (the data is a pure function of these)."""
    from gen import Batch, Params, make, seed_for
    idx = {"C1": 0, "C2": 1, "C3": 2, "C4": 3}[config]
    seed = seed_for(idx) + seed
    params = Params(k_start=21, k_min=21, k_max=21) if config == "C1" else Params()
    path = os.path.join(CACHE, f"{config}_{seed}_{scale}.npz")
    if os.path.exists(path):
        try:
            return Batch.load(path), params
        except Exception:
            pass
    kw = {"scale": scale} if config in ("C2", "C4") else {}
    t = time.time()
    b = make(config, seed=seed, **kw)
    log(f"[bench] generated {config} seed {seed}: {b.n_contigs} contigs, {b.n_reads} reads in {time.time() - t:.1f}s")
    try:
        os.makedirs(CACHE, exist_ok=True)
        tmp = path + f".{os.getpid()}.tmp.npz"
        b.save(tmp)
        os.replace(tmp, path)
    except OSError:
        pass
    return b, params


class ClockSampler:
    """nvidia-smi clocks / throttle reasons during the timed region (B200_PROFILING.md)."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu):
        self.gpu = gpu
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            out, _ = self.proc.communicate(timeout=10)
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in getattr(self, "lines", []):
            f = [x.strip() for x in l.split(",")]
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except (ValueError, IndexError):
                continue
            for n, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


def flush_l2(buf):
    buf.add_(1)   # write 256 MB (> 126 MB L2) between timed steps


def roofline_peaks():
    """Measured denominators: HBM from MEASURED_PEAKS.json (driver-written), the shared-memory
    random-update rate from our microbenchmark (profiles/micro_random_update.json)."""
    peaks = {}
    try:
        peaks["hbm_gbs"] = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
        peaks["hbm_src"] = "MEASURED_PEAKS.json"
    except Exception:
        peaks["hbm_gbs"] = 6650.0
        peaks["hbm_src"] = "fallback (B200_PROFILING.md)"
    try:
        m = json.load(open(os.path.join(ROOT, "profiles", "micro_random_update.json")))
        peaks["smem_gups"] = m["smem_atomic_add32"]
        peaks["insert_gups"] = m.get("smem_hash_insert")
        peaks["smem_src"] = "profiles/micro_random_update.json (smem_atomic_add32, measured on B200)"
    except Exception:
        peaks["smem_gups"] = None
        peaks["smem_src"] = "unmeasured"
    return peaks


def cpu_oracle_sample(batch, params, budget_s=15.0, seed=0, cores=None):
    """Time the oracle (as it stands: single-threaded C++) on a bounded random sample of the
    workload's ends, one process per host core.  Returns (bases/s, ends/s, cores, sample desc)."""
    import multiprocessing as mp
    import oracle
    oracle.build()
    cores = cores or os.cpu_count() or 1
    rng = np.random.default_rng(seed)
    ends = rng.permutation(batch.n_ends)
    # calibrate on a small slice, then size the sample to ~budget_s of all-core CPU time
    cal = ends[:64]
    t = time.time()
    r = oracle.extend(batch, params, ends=cal)
    dt = max(time.time() - t, 1e-3)
    per_end = dt / len(cal)
    n = int(min(batch.n_ends, max(len(cal), budget_s * cores / per_end)))
    sample = ends[:n]
    chunks = np.array_split(sample, cores)
    global _ORC_BATCH, _ORC_PARAMS
    _ORC_BATCH, _ORC_PARAMS = batch, params
    ctx = mp.get_context("fork")
    t = time.time()
    with ctx.Pool(cores) as pool:
        outs = pool.map(_oracle_chunk, chunks)
    wall = time.time() - t
    bases = sum(o[0] for o in outs)
    return bases / wall, n / wall, cores, (f"{n} random ends of {batch.n_ends} (seed {seed}), "
                                           f"{cores} processes x single-thread oracle, {wall:.1f}s wall")


_ORC_BATCH = _ORC_PARAMS = None


def _oracle_chunk(ends):
    import oracle
    if len(ends) == 0:
        return (0, 0)
    r = oracle.extend(_ORC_BATCH, _ORC_PARAMS, ends=ends)
    return (sum(len(x) for x in r["ext"]), len(ends))


def dist_init(n_gpus):
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return rank, world, local


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def run_reference(args):
    """Reference arm = the CPU oracle on this arm's config/metric, each step a bounded sample."""
    rank = int(os.environ.get("RANK", 0))
    if rank != 0:
        return 0
    batch, params = load_workload(args.config, 0, args.scale)
    if args.k_start:
        params = params.replace(k_start=args.k_start, k_min=min(params.k_min, args.k_start),
                                k_max=max(params.k_max, args.k_start))
    vals = []
    for step in range(args.warmup + args.steps):
        v, eps, cores, desc = cpu_oracle_sample(batch, params, budget_s=args.ref_budget, seed=step)
        if step >= args.warmup:
            vals.append((v, eps, desc))
    v = statistics.median([x[0] for x in vals])
    eps = statistics.median([x[1] for x in vals])
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": CONFIG_DESC[args.config] + (f", k_start={args.k_start}" if args.k_start else ""),
                       "n_ends": batch.n_ends, "n_reads": batch.n_reads},
            "contig_ends_per_s": eps,
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": os.cpu_count(), "kind": "oracle",
                             "sample": vals[-1][2]},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4", choices=["C1", "C2", "C3", "C4"])
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-budget", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunks", type=int, default=8)
    ap.add_argument("--k-start", type=int, default=None,
                    help="NEXT N2: LA at another k of the assembler's contig iteration (21, 33, 55, 77)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    from paper_conf_sc_awanhedbdoy21_b200.build import build
    rank, world, local = dist_init(args.gpus)
    if rank == 0:
        build()
    barrier(world)
    torch.cuda.set_device(local)
    batch, params = load_workload(args.config, rank, args.scale)
    if args.k_start:
        params = params.replace(k_start=args.k_start, k_min=min(params.k_min, args.k_start),
                                k_max=max(params.k_max, args.k_start))
    stream = torch.cuda.Stream()
    la = LocalAssembler(local, stream=stream)

    # ---------------- device-resident timing (kernel path) ----------------
    dev = type("DevBatch", (), {})()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
        setattr(dev, f, torch.from_numpy(getattr(batch, f)).to(f"cuda:{local}"))
    la.load(dev, params)
    flush = torch.zeros(64 << 20, dtype=torch.float32, device=f"cuda:{local}")
    for _ in range(args.warmup):
        la.extend_device()
    torch.cuda.synchronize()
    stats = []
    evs = []
    barrier(world)
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            with torch.cuda.stream(stream):
                flush_l2(flush)
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream)
            la.extend_device()
            e1.record(stream)
            evs.append((e0, e1))
            stats.append(la.stats())
        torch.cuda.synchronize()
    barrier(world)
    step_ms = [a.elapsed_time(b) for a, b in evs]
    ms_total = sum(step_ms)
    bases = stats[-1]["ext_bases"]
    ends = batch.n_ends
    ms_max = max_over_ranks(ms_total, world)
    bases_all = sum_over_ranks(bases * args.steps, world)
    ends_all = sum_over_ranks(ends * args.steps, world)
    value = bases_all / (ms_max / 1e3)
    ends_per_s = ends_all / (ms_max / 1e3)
    st = stats[-1]
    ms_smem = statistics.mean(s["ms_smem"] for s in stats)
    launches = sum(s["kernel_launches"] for s in stats)

    # ---------------- NEXT N1: on-device append of the extensions (not part of the step) ----------------
    d = la.extend_device()
    ap_ms = []
    for i in range(6):
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        la.append_extensions(dev.contig_seq, dev.contig_off, d["ext_off"], d["ext_seq"])
        a1.record(stream)
        a1.synchronize()
        if i:
            ap_ms.append(a0.elapsed_time(a1))
    ap_bytes = 2 * (int(batch.contig_off[-1] - batch.contig_off[0]) + int(la.stats()["ext_bases"])) + \
        8 * (4 * batch.n_contigs + 3)
    ap_med = statistics.median(ap_ms)
    append_n1 = {"kernel": "k_append_ext", "ms": ap_med, "bound": "hbm", "algorithmic_bytes": ap_bytes,
                 "achieved": ap_bytes / (ap_med / 1e3) / 1e9, "unit": "GB/s",
                 "note": "la_append_extensions on this step's results, CUDA events around the call (includes "
                         "its launch); outside the timed step; DESIGN.md §10a"}

    # ---------------- end to end through the public API (host buffers) ----------------
    e2e = None
    if not args.no_e2e:
        pinned = type("HostBatch", (), {})()
        h2d = 0
        for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
            t = torch.from_numpy(getattr(batch, f)).pin_memory()
            setattr(pinned, f, t)
            h2d += t.numel() * t.element_size()
        la2 = LocalAssembler(local, stream=stream)
        la2.extend_streamed(pinned, params, args.e2e_chunks)      # warm-up (allocations)
        torch.cuda.synchronize()
        barrier(world)
        t0 = time.perf_counter()
        d2h = 0
        e2e_steps = max(1, min(args.steps, 3))
        for _ in range(e2e_steps):
            r = la2.extend_streamed(pinned, params, args.e2e_chunks)
            d2h = r.ext_off.nbytes + r.ext_seq.nbytes + r.term.nbytes + r.k_used.nbytes + r.n_attempts.nbytes
        torch.cuda.synchronize()
        el = max_over_ranks(time.perf_counter() - t0, world)
        e2e = {"value": sum_over_ranks(r.ext_off[-1] * e2e_steps, world) / el, "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": el / e2e_steps * 1e3, "timing": "host wall clock around la_extend_streamed, max over ranks",
               "api": f"la_extend_streamed(host pinned batch, {args.e2e_chunks} chunks): H2D of chunk i+1 "
                      "overlaps encode+extend of chunk i; results D2H into host memory"}
        la2.close()

    # ---------------- result gather (after timing; the only inter-GPU traffic) ----------------
    gather_ms = None
    if world > 1:
        from paper_conf_sc_awanhedbdoy21_b200.dist import gather_results
        res = la.extend()
        torch.cuda.synchronize()
        barrier(world)
        t0 = time.perf_counter()
        gather_results(res, np.arange(batch.n_contigs, dtype=np.int64) + rank * batch.n_contigs,
                       batch.n_contigs * world)
        barrier(world)
        gather_ms = (time.perf_counter() - t0) * 1e3

    if rank != 0:
        la.close()
        return 0
    peaks = roofline_peaks()
    roof = None
    hbm_bytes_alg = int(batch.read_seq.nbytes) // 4 * 2   # packed reads (2-bit seq + 2-bit qual) streamed once per step
    if peaks["smem_gups"]:
        ach = st["inserts_smem"] / (ms_smem / 1e3) / 1e9 if ms_smem > 0 else 0.0
        traffic, tsrc = None, None
        try:   # DRAM bytes per step of the table kernels from the committed ncu capture (tools/traffic.py)
            tj = json.load(open(os.path.join(ROOT, "profiles", "r01_traffic.json")))
            traffic = tj["table_kernels_per_step"]["dram_bytes"]
            tsrc = "profiles/r01_traffic.json (ncu dram__bytes_read.sum + dram__bytes_write.sum, table kernels, per step)"
        except Exception:
            pass
        roof = {"bound": "smem", "kernel": "k_small / k_smem (table build + link + walk, all classes)",
                "achieved": ach, "peak": peaks["smem_gups"], "unit": "G updates/s",
                "frac": ach / peaks["smem_gups"], "traffic": traffic, "traffic_src": tsrc,
                "algorithmic_bytes": hbm_bytes_alg,
                "peak_src": peaks["smem_src"],
                "note": "algorithmic unit = one vote insert (1 random table update); see DESIGN.md §7"}
    hbm_bytes = int(batch.read_seq.nbytes) // 4 * 2   # packed reads (2-bit seq + 2-bit qual) streamed once per step
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": CONFIG_DESC[args.config] + (f", k_start={args.k_start}" if args.k_start else ""),
                   "k_schedule": [params.k_start, params.k_min, params.k_max, params.k_shift],
                   "n_ends": batch.n_ends, "n_contigs": batch.n_contigs,
                   "n_reads": batch.n_reads, "scale": args.scale, "seed": "20211114+cfg+rank",
                   "l2": "flushed between timed steps (256 MB write)", "parallelism": f"contig-shards x{world}"},
        "contig_ends_per_s": ends_per_s,
        "ends_with_reads_per_s": (ends - st["ends_by_class"][0]) * world * args.steps / (ms_max / 1e3),
        "step_ms": step_ms,
        "phase_ms": {"smem_kernel": ms_smem, "smem_large_tables": statistics.mean(s["ms_smem_medium"] for s in stats),
                     "global_rounds": statistics.mean(s["ms_global"] for s in stats),
                     "emit": statistics.mean(s["ms_emit"] for s in stats)},
        "work": {"inserts": st["inserts"], "walk_steps": st["walk_steps"], "attempts": st["attempts"],
                 "ext_bases": st["ext_bases"], "ends_by_class": st["ends_by_class"],
                 "global_rounds": st["global_rounds"], "ends_medium": st["ends_medium"], "ends_xl": st["ends_xl"],
                 "inserts_smem": st["inserts_smem"],
                 "classes": {n: {"ends": st["cls_ends"][i], "inserts": st["cls_inserts"][i],
                                 "attempts": st["cls_attempts"][i], "filtered": st["cls_filtered"][i],
                                 "ms": round(st["cls_ms"][i], 3)}
                             for i, n in enumerate(["smem64x12", "smem128x6", "smem256x3", "smem512x2",
                                                    "smem1024x1", "xl1024x1"])}},
        "roofline": roof,
        "roofline_insert": ({"bound": "smem", "kernel": roof["kernel"], "achieved": roof["achieved"],
                             "peak": peaks["insert_gups"], "unit": "G inserts/s",
                             "frac": roof["achieved"] / peaks["insert_gups"],
                             "peak_src": "profiles/micro_random_update.json smem_hash_insert: the table's insert "
                                         "primitive alone (hash + slot-pair probe + vote atomic), measured on B200"}
                            if roof and peaks.get("insert_gups") else None),
        "roofline_hbm": {"bound": "hbm", "achieved": hbm_bytes / (ms_max / args.steps / 1e3) / 1e9,
                         "peak": peaks["hbm_gbs"], "unit": "GB/s",
                         "frac": hbm_bytes / (ms_max / args.steps / 1e3) / 1e9 / peaks["hbm_gbs"],
                         "peak_src": peaks["hbm_src"], "traffic": None},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "e2e": e2e,
        "gather_ms": gather_ms,
        "append_n1": dict(append_n1, peak=peaks["hbm_gbs"], frac=append_n1["achieved"] / peaks["hbm_gbs"]),
    }
    if not args.no_cpu_baseline and world == 1:
        v, eps, cores, desc = cpu_oracle_sample(batch, params, budget_s=args.ref_budget)
        line["cpu_baseline"] = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc,
                                "ends_per_s": eps}
    print(json.dumps(line), flush=True)
    la.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
