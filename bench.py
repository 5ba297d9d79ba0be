#!/usr/bin/env python
"""Benchmark of the B200 local-assembly hot path.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl ours|reference]
                  [--scaling strong|weak] [--k-start K]

A step = one la_extend over the whole batch: plan, the table-class kernels (build + ext rule + walk
+ k retry for every end that fits shared memory or the XL scratch), the global-memory rounds for
the rest, compaction.  `value` = extended bases/s with the inputs resident in HBM (device-timed with
CUDA events on the library's stream, max over ranks); `e2e` = the same metric through the public API
from pinned host buffers (H2D + encode + extend + D2H of all results inside the timed region).

N > 1: `--gpus N` re-launches itself under torch.distributed.run (one process per GPU).  Default
`--scaling strong` is SURVEY §8(d) C5: every rank maps the same C4 batch, takes its contigs from the
shared deterministic partition (dist.partition: LPT for the heaviest 1% + contiguous fill), extends
only those, and the results are gathered to rank 0 once after the timed region (the only inter-GPU
traffic, `gather_ms`).  `--scaling weak`: every rank extends its own independent C4 sample.

Every run checks its own parity (`parity`): the CPU oracle recomputes a random sample of the
benchmarked batch's ends and they must equal the GPU step's results end by end (extension, term,
k_used, attempts); a mismatch makes the bench exit non-zero.
The reference arm (--impl reference) is the CPU oracle (oracle/), timed on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import shutil
import socket
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
    "C4": "C4 paper-shaped batch (500-species metagenome, lognormal(0,1.5), 150 bp pairs, ~1M contigs) on 1 B200",
    "C4S": "C4S = r01's C4 (500-species metagenome, 510k contigs, 31.7M read copies)",
    "C4F": "C4F = C4's contigs with the paper's Fig 3 mix of reads per end (70% none, 29% 1-9, 1% all)",
}
CACHE = os.environ.get("LA_GEN_CACHE", "/tmp/la_gen_cache")
FIELDS = ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off")
CLASS_NAMES = ["smem64x12", "smem128x6", "smem256x3", "smem512x2", "smem1024x1", "xl1024x1", "xlc2x1024"]
# The paper's own numbers, with their hardware: context, not the target.
PAPER = {
    "context_not_target": True,
    "la_speedup_gpu_vs_cpu_la": {
        "value": "about 7x (\"more than 7x\")",
        "hardware": "64 Summit nodes; GPU LA on 6x V100 16 GB per node vs CPU LA on 2x POWER9 per node (all cores)",
        "workload": "WA marine metagenome, 2,465,328,090 paired 150 bp reads (813 GB)",
        "cite": "PAPER.md:28-30, 1027-1031 (Fig 13)"},
    "la_speedup_1024_nodes": {"value": "2.65x", "hardware": "1024 Summit nodes", "cite": "PAPER.md:1031-1035"},
    "end_to_end_gain": {"value": "42% (2128 s -> 1495 s)", "hardware": "64 Summit nodes",
                        "cite": "PAPER.md:28-30, 1090-1093 (Fig 14)"},
    "la_share_of_pipeline": {"value": "34% (CPU LA) -> 6% (GPU LA)", "cite": "PAPER.md:367-370, 1106-1108"},
    "note": "the paper publishes no absolute LA throughput (bases/s, ends/s); its ratios compare whole "
            "Summit nodes, so no vs_baseline is computed",
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------------------------------------
# workloads: deterministic, cached as one .npy per array so that other ranks can memory-map them
# ------------------------------------------------------------------------------------------------
def workload_params(config):
    from gen import Params
    return Params(k_start=21, k_min=21, k_max=21) if config == "C1" else Params()


def _cache_dir(config, seed, scale):
    from gen.synth import GEN_VERSION
    return os.path.join(CACHE, f"{config}_{seed}_{scale}_v{GEN_VERSION}")


def load_workload(config, seed, scale, mmap=False):
    """(batch, params) of a deterministic synthetic workload (a pure function of config, seed,
    scale), cached on local disk; mmap=True maps the cached arrays read-only instead of loading."""
    from gen import Batch, make, seed_for
    idx = {"C1": 0, "C2": 1, "C3": 2, "C4": 3, "C4S": 3, "C4F": 3}[config]
    seed = seed_for(idx) + seed
    d = _cache_dir(config, seed, scale)
    if os.path.exists(os.path.join(d, "ok")):
        try:
            arrs = [np.load(os.path.join(d, f + ".npy"), mmap_mode="r" if mmap else None) for f in FIELDS]
            return Batch(*arrs), workload_params(config)
        except Exception:
            pass
    kw = {"scale": scale} if config in ("C2", "C4", "C4S", "C4F") else {}
    t = time.time()
    b = make(config, seed=seed, **kw)
    log(f"[bench] generated {config} seed {seed}: {b.n_contigs} contigs, {b.n_reads} reads in {time.time() - t:.1f}s")
    try:
        tmp = d + f".{os.getpid()}.tmp"
        os.makedirs(tmp, exist_ok=True)
        for f in FIELDS:
            np.save(os.path.join(tmp, f + ".npy"), getattr(b, f))
        open(os.path.join(tmp, "ok"), "w").close()
        shutil.rmtree(d, ignore_errors=True)
        os.replace(tmp, d)
    except OSError:
        pass
    if mmap:
        return load_workload(config, seed - seed_for(idx), scale, mmap=True)
    return b, workload_params(config)


def fig3_bins(batch):
    """Share of ends per read-count bin of the paper's Fig 3: 0, 1-9, >= 10 reads."""
    r = np.diff(np.asarray(batch.end_read_off))
    n = max(r.shape[0], 1)
    return {"0": float((r == 0).sum() / n), "1-9": float(((r > 0) & (r < 10)).sum() / n),
            ">=10": float((r >= 10).sum() / n), "reads_per_end_median": float(np.median(r)) if r.size else 0.0,
            "reads_per_end_p99": float(np.percentile(r, 99)) if r.size else 0.0,
            "reads_per_end_max": int(r.max()) if r.size else 0,
            "paper": "majority 0, 10-30% 1-9, <1% >=10 (arcticsynth LA input); reported, not enforced"}


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
    """Measured denominators: HBM from MEASURED_PEAKS.json (driver-written); the shared-memory and
    L2 random-update rates from our microbenchmark (profiles/micro_random_update.json)."""
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
        peaks["l2_gups"] = m["global_red_l2"]
        peaks["smem_src"] = "profiles/micro_random_update.json (smem_atomic_add32 / global_red_l2, measured on B200)"
    except Exception:
        peaks["smem_gups"] = peaks["l2_gups"] = None
        peaks["smem_src"] = "unmeasured"
    return peaks


# ------------------------------------------------------------------------------------------------
# the CPU oracle: timed baseline + parity sample
# ------------------------------------------------------------------------------------------------
_ORC_BATCH = _ORC_PARAMS = None


def _oracle_chunk(ends):
    import oracle
    if len(ends) == 0:
        return None
    return oracle.extend(_ORC_BATCH, _ORC_PARAMS, ends=ends)


def oracle_sample(batch, params, budget_s=15.0, seed=0, cores=None, min_ends=0):
    """Run the oracle (as it stands: single-threaded C++, one process per host core) on a bounded
    random sample of the batch's ends.  Returns the timing and the per-end results."""
    import multiprocessing as mp
    import oracle
    oracle.build()
    cores = cores or os.cpu_count() or 1
    rng = np.random.default_rng(seed)
    ends = rng.permutation(batch.n_ends)
    cal = ends[:64]
    t = time.time()
    oracle.extend(batch, params, ends=cal)
    per_end = max(time.time() - t, 1e-3) / len(cal)
    n = int(min(batch.n_ends, max(len(cal), min_ends, budget_s * cores / per_end)))
    sample = np.sort(ends[:n])
    chunks = np.array_split(sample, cores)
    global _ORC_BATCH, _ORC_PARAMS
    _ORC_BATCH, _ORC_PARAMS = batch, params
    ctx = mp.get_context("fork")
    t = time.time()
    with ctx.Pool(cores) as pool:
        outs = [o for o in pool.map(_oracle_chunk, chunks) if o is not None]
    wall = time.time() - t
    res = {"ends": np.concatenate([o["ends"] for o in outs]), "ext": [x for o in outs for x in o["ext"]],
           "term": np.concatenate([o["term"] for o in outs]), "k_used": np.concatenate([o["k_used"] for o in outs]),
           "n_attempts": np.concatenate([o["n_attempts"] for o in outs])}
    bases = sum(len(x) for x in res["ext"])
    desc = f"{n} random ends of {batch.n_ends} (seed {seed}), {cores} processes x single-thread oracle, {wall:.1f}s wall"
    return {"value": bases / wall, "ends_per_s": n / wall, "cores": cores, "sample": desc, "res": res}


def parity_check(result, ref):
    """GPU result (host Result of the benchmarked batch) vs the oracle's results on the sampled ends:
    extension string, termination code, k of the returned walk and attempts, end by end."""
    ends = ref["ends"]
    off, seq = result.ext_off, result.ext_seq
    bad = []
    for i, e in enumerate(ends.tolist()):
        if (seq[off[e]:off[e + 1]].tobytes() != ref["ext"][i].encode() or result.term[e] != ref["term"][i]
                or result.k_used[e] != ref["k_used"][i] or result.n_attempts[e] != ref["n_attempts"][i]):
            bad.append(e)
    out = {"ends_checked": int(ends.shape[0]), "mismatches": len(bad),
           "fields": "extension string, term, k_used, n_attempts (bit-exact)",
           "reference": "oracle/ (CPU, single-threaded C++) on the sampled ends of the benchmarked batch"}
    if bad:
        e = bad[0]
        i = int(np.nonzero(ends == e)[0][0])
        out["first_mismatch"] = {"end": e, "gpu": [seq[off[e]:off[e + 1]].tobytes().decode()[:60], int(result.term[e]),
                                                   int(result.k_used[e]), int(result.n_attempts[e])],
                                 "oracle": [ref["ext"][i][:60], int(ref["term"][i]), int(ref["k_used"][i]),
                                            int(ref["n_attempts"][i])]}
    return out


# ------------------------------------------------------------------------------------------------
# torch.distributed plumbing (one process per GPU)
# ------------------------------------------------------------------------------------------------
class Dist:
    def __init__(self):
        self.rank = int(os.environ.get("RANK", 0))
        self.world = int(os.environ.get("WORLD_SIZE", 1))
        self.local = int(os.environ.get("LOCAL_RANK", 0))
        self.backend = None
        self.device = 0

    def init(self):
        import torch
        ndev = max(torch.cuda.device_count(), 1)
        self.device = self.local % ndev
        torch.cuda.set_device(self.device)
        if self.world > 1:
            import torch.distributed as dist
            # NCCL refuses two ranks on one GPU: when ranks share a device (a 2-rank check on a
            # 1-GPU box) the control plane (barrier, max, gather) runs over gloo instead
            self.backend = "nccl" if ndev >= self.world else "gloo"
            if self.backend == "nccl":
                dist.init_process_group("nccl", device_id=torch.device("cuda", self.device))
            else:
                dist.init_process_group("gloo")
        return self

    def _t(self, x, dtype):
        import torch
        dev = f"cuda:{self.device}" if self.backend == "nccl" else "cpu"
        return torch.tensor([x], dtype=dtype, device=dev)

    def reduce(self, x, op):
        if self.world == 1:
            return x
        import torch
        import torch.distributed as dist
        t = self._t(x, torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
        return float(t.item())

    def barrier(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.barrier()


def relaunch_under_torchrun(args):
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    log("[bench] --gpus", args.gpus, "-> relaunching as:", " ".join(cmd))
    os.execv(sys.executable, cmd)


# ------------------------------------------------------------------------------------------------
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
        o = oracle_sample(batch, params, budget_s=args.ref_budget, seed=step)
        if step >= args.warmup:
            vals.append(o)
    v = statistics.median([x["value"] for x in vals])
    eps = statistics.median([x["ends_per_s"] for x in vals])
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True,
            "scaling": "strong" if args.scaling == "strong" else "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": CONFIG_DESC[args.config] + (f", k_start={args.k_start}" if args.k_start else ""),
                       "n_ends": batch.n_ends, "n_reads": batch.n_reads},
            "contig_ends_per_s": eps,
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": vals[-1]["cores"], "kind": "oracle",
                             "sample": vals[-1]["sample"]},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4", choices=["C1", "C2", "C3", "C4", "C4S", "C4F"])
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="N>1: strong = C5, one C4 batch partitioned over the ranks; weak = a sample per rank")
    ap.add_argument("--ref-budget", type=float, default=15.0)
    ap.add_argument("--parity-min-ends", type=int, default=300000,
                    help="minimum number of oracle-checked ends (capped by the batch)")
    ap.add_argument("--no-cpu-baseline", action="store_true", help="skip the oracle (timing and parity)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-select", action="store_true", help="skip the NEXT N4 selection block")
    ap.add_argument("--no-replay", action="store_true", help="skip the build-only replay (roofline_build)")
    ap.add_argument("--e2e-chunks", type=int, default=8)
    ap.add_argument("--coexec-share", type=float, default=0.05,
                    help="NEXT N3 measurement: share of the smallest class's ends on host threads (0: skip)")
    ap.add_argument("--coexec-threads", type=int, default=0, help="host threads for N3 (0: cores - 2)")
    ap.add_argument("--k-start", type=int, default=None,
                    help="NEXT N2: LA at another k of the assembler's contig iteration (21, 33, 55, 77)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch_under_torchrun(args)
    if int(os.environ.get("WORLD_SIZE", 1)) != args.gpus:
        log(f"[bench] WORLD_SIZE={os.environ.get('WORLD_SIZE')} but --gpus {args.gpus}: refusing to run")
        return 2

    import torch
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    from paper_conf_sc_awanhedbdoy21_b200.build import build
    from paper_conf_sc_awanhedbdoy21_b200.dist import contig_work, gather_results, partition
    D = Dist().init()
    rank, world, dev_i = D.rank, D.world, D.device
    if rank == 0:
        build()
    strong = args.scaling == "strong"
    # the batch: rank 0 generates (or finds) the cached workload first, the others map it
    if rank == 0 or not strong:
        full, params = load_workload(args.config, 0 if strong else rank, args.scale, mmap=world > 1)
    D.barrier()
    if rank != 0 and strong:
        full, params = load_workload(args.config, 0, args.scale, mmap=True)
    if args.k_start:
        params = params.replace(k_start=args.k_start, k_min=min(params.k_min, args.k_start),
                                k_max=max(params.k_max, args.k_start))
    if world > 1 and strong:
        owner = partition(contig_work(full, params.k_start), world)
        mine = np.nonzero(owner == rank)[0].astype(np.int64)
        batch = full.select_contigs(mine)
    else:
        mine = np.arange(full.n_contigs, dtype=np.int64)
        batch = full
    stream = torch.cuda.Stream()
    la = LocalAssembler(dev_i, stream=stream)

    # ---------------- device-resident timing (kernel path) ----------------
    dev = type("DevBatch", (), {})()
    for f in FIELDS:
        setattr(dev, f, torch.from_numpy(np.ascontiguousarray(getattr(batch, f))).to(f"cuda:{dev_i}"))
    la.load(dev, params)
    flush = torch.zeros(64 << 20, dtype=torch.float32, device=f"cuda:{dev_i}")
    for _ in range(args.warmup):
        la.extend_device()
    torch.cuda.synchronize()
    stats, evs = [], []
    D.barrier()
    torch.cuda.synchronize()
    with ClockSampler(dev_i) as clk:
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
    D.barrier()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    ms_total = sum(step_ms)
    st = stats[-1]
    bases = st["ext_bases"]
    ms_max = D.reduce(ms_total, "max")
    bases_all = D.reduce(bases * args.steps, "sum")
    ends_all = D.reduce(batch.n_ends * args.steps, "sum")
    value = bases_all / (ms_max / 1e3)
    ends_per_s = ends_all / (ms_max / 1e3)
    ms_smem = statistics.mean(s["ms_smem"] for s in stats)
    launches = sum(s["kernel_launches"] for s in stats)

    # ---------------- hash-build phase: build-only replay of the recorded attempts ----------------
    replay = None
    if not args.no_replay:
        rms = []
        for i in range(4):
            with torch.cuda.stream(stream):
                flush_l2(flush)
            la.replay_build()
            if i:
                rms.append(la.stats())
        replay = rms

    # ---------------- NEXT N3: CPU+GPU co-execution (outside the timed step) ----------------
    n3 = None
    if args.coexec_share > 0:
        thr = args.coexec_threads or max(1, (os.cpu_count() or 2) - 2)
        la.set_coexec(thr, args.coexec_share)
        ms3 = []
        for i in range(4):
            with torch.cuda.stream(stream):
                flush_l2(flush)
                a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a0.record(stream)
            la.extend_device()
            a1.record(stream)
            a1.synchronize()
            if i:
                ms3.append(a0.elapsed_time(a1))
        st3 = la.stats()
        la.set_coexec(0, 0.0)
        m3 = statistics.median(ms3)
        n3 = {"host_threads": thr, "share_of_smallest_class": args.coexec_share, "host_ends": st3["cpu_ends"],
              "host_inserts": st3["cpu_inserts"], "ms_per_step": m3, "gpu_only_ms_per_step": ms_total / args.steps,
              "value": st3["ext_bases"] / (m3 / 1e3), "unit": UNIT,
              "note": "la_set_coexec: the lightest ends of the smallest class on host threads while the GPU "
                      "runs (NEXT N3, paper §4.3); this rank, CUDA events around la_extend_device, outside "
                      "the timed step; DESIGN.md §10c"}

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
    del dev
    torch.cuda.empty_cache()

    # ---------------- NEXT N4: candidate-read selection (not part of the step) ----------------
    select_n4 = None
    if not args.no_select and rank == 0:
        select_n4 = bench_select(dev_i, stream)
        torch.cuda.empty_cache()

    # ---------------- end to end through the public API (host buffers) ----------------
    e2e = None
    if not args.no_e2e:
        pinned = type("HostBatch", (), {})()
        h2d = 0
        for f in FIELDS:
            t = torch.from_numpy(np.ascontiguousarray(getattr(batch, f))).pin_memory()
            setattr(pinned, f, t)
            h2d += t.numel() * t.element_size()
        la2 = LocalAssembler(dev_i, stream=stream)
        la2.extend_streamed(pinned, params, args.e2e_chunks)      # warm-up (allocations)
        torch.cuda.synchronize()
        D.barrier()
        t0 = time.perf_counter()
        d2h = 0
        e2e_steps = max(1, min(args.steps, 3))
        for _ in range(e2e_steps):
            r = la2.extend_streamed(pinned, params, args.e2e_chunks)
            d2h = r.ext_off.nbytes + r.ext_seq.nbytes + r.term.nbytes + r.k_used.nbytes + r.n_attempts.nbytes
        torch.cuda.synchronize()
        el = D.reduce(time.perf_counter() - t0, "max")
        e2e = {"value": D.reduce(int(r.ext_off[-1]) * e2e_steps, "sum") / el, "unit": UNIT,
               "h2d_bytes_per_step": int(D.reduce(h2d, "sum")), "d2h_bytes_per_step": int(D.reduce(d2h, "sum")),
               "ms_per_step": el / e2e_steps * 1e3, "timing": "host wall clock around la_extend_streamed, max over ranks",
               "api": f"la_extend_streamed(host pinned batch, {args.e2e_chunks} chunks): H2D of chunk i+1 "
                      "overlaps encode+extend of chunk i; results D2H into host memory"}
        la2.close()
        del pinned

    # ---------------- results on the host; gather to rank 0 (the only inter-GPU traffic) ----------------
    res = la.extend()
    gather_ms = None
    if world > 1 and strong:
        D.barrier()
        t0 = time.perf_counter()
        res = gather_results(res, mine, full.n_contigs)
        D.barrier()
        gather_ms = (time.perf_counter() - t0) * 1e3
    la.close()
    if rank != 0:
        return 0

    # ---------------- parity of this run (oracle sample of the benchmarked batch) + cpu_baseline ----------------
    parity, cpu = None, None
    check_batch = full if (world == 1 or strong) else batch
    if not args.no_cpu_baseline:
        o = oracle_sample(check_batch, params, budget_s=args.ref_budget if world == 1 else args.ref_budget / 2,
                          min_ends=args.parity_min_ends)
        parity = parity_check(res, o["res"])
        if world == 1:
            cpu = {"value": o["value"], "unit": UNIT, "cores": o["cores"], "kind": "oracle", "sample": o["sample"],
                   "ends_per_s": o["ends_per_s"]}

    peaks = roofline_peaks()
    roof, roof_build = None, None
    inserts = st["inserts_smem"]
    if peaks["smem_gups"] and ms_smem > 0:
        # whole table phase (build + link + walk + scheduling) against the shared-memory update peak
        ach = inserts / (ms_smem / 1e3) / 1e9
        roof = {"bound": "smem", "kernel": "table-class kernels, whole step (build + link + walk)",
                "achieved": ach, "peak": peaks["smem_gups"], "unit": "G updates/s", "frac": ach / peaks["smem_gups"],
                "traffic": None, "peak_src": peaks["smem_src"],
                "note": "algorithmic unit = one vote insert (1 random table update); DESIGN.md §7"}
    if replay and peaks["smem_gups"]:
        roof_build = build_roofline(replay, peaks)
        if roof is not None:
            roof["traffic"] = roof_build.get("traffic")
    hbm_bytes = int(np.asarray(batch.read_off)[-1]) // 4 * 2   # packed reads (2-bit seq + 2-bit qual), once per step
    cls = {n: {"ends": st["cls_ends"][i], "inserts": st["cls_inserts"][i], "attempts": st["cls_attempts"][i],
               "filtered": st["cls_filtered"][i], "ms": round(st["cls_ms"][i], 3)} for i, n in enumerate(CLASS_NAMES)}
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": CONFIG_DESC[args.config] + (f", k_start={args.k_start}" if args.k_start else ""),
                   "k_schedule": [params.k_start, params.k_min, params.k_max, params.k_shift],
                   "n_ends": full.n_ends if strong else batch.n_ends * world,
                   "n_contigs": full.n_contigs if strong else batch.n_contigs * world,
                   "n_reads": full.n_reads if strong else batch.n_reads * world, "scale": args.scale,
                   "seed": "20211114+cfg" + ("" if strong else "+rank"), "fig3_bins": fig3_bins(full),
                   "l2": "flushed between timed steps (256 MB write)",
                   "parallelism": (f"C5: one batch partitioned over {world} ranks (LPT top 1% + contiguous fill)"
                                   if strong else f"independent samples x{world}") + f", backend {D.backend or 'none'}"},
        "contig_ends_per_s": ends_per_s,
        "ends_with_reads_per_s": D.reduce((batch.n_ends - st["ends_by_class"][0]) * args.steps, "sum") / (ms_max / 1e3)
        if world == 1 else None,
        "step_ms": step_ms,
        "phase_ms": {"table_kernels": ms_smem, "global_rounds": statistics.mean(s["ms_global"] for s in stats),
                     "emit": statistics.mean(s["ms_emit"] for s in stats),
                     "build_replay": roof_build["ms"] if roof_build else None},
        "work": {"inserts": st["inserts"], "walk_steps": st["walk_steps"], "attempts": st["attempts"],
                 "ext_bases": st["ext_bases"], "ends_by_class": st["ends_by_class"],
                 "global_rounds": st["global_rounds"], "ends_xl": st["ends_xl"], "inserts_smem": inserts,
                 "attempts_hist": st["attempts_hist"], "classes": cls},
        "roofline": roof,
        "roofline_build": roof_build,
        "roofline_hbm": {"bound": "hbm", "achieved": hbm_bytes / (ms_max / args.steps / 1e3) / 1e9,
                         "peak": peaks["hbm_gbs"], "unit": "GB/s",
                         "frac": hbm_bytes / (ms_max / args.steps / 1e3) / 1e9 / peaks["hbm_gbs"],
                         "peak_src": peaks["hbm_src"], "traffic": None,
                         "note": "packed read bytes streamed once per step: the path is not HBM-bound"},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "e2e": e2e,
        "gather_ms": gather_ms,
        "parity": parity,
        "append_n1": dict(append_n1, peak=peaks["hbm_gbs"], frac=append_n1["achieved"] / peaks["hbm_gbs"]),
        "coexec_n3": n3,
        "select_n4": select_n4,
        "paper": PAPER,
    }
    if cpu:
        line["cpu_baseline"] = cpu
    print(json.dumps(line), flush=True)
    if parity and parity["mismatches"]:
        log(f"[bench] PARITY FAILURE: {parity['mismatches']} of {parity['ends_checked']} sampled ends differ "
            f"from the oracle: {parity.get('first_mismatch')}")
        return 1
    if select_n4 and select_n4.get("parity", {}).get("arrays_differing", 0):
        log(f"[bench] N4 PARITY FAILURE: {select_n4['parity']}")
        return 1
    return 0


def bench_select(dev_i, stream):
    """NEXT N4 (la_select_reads): candidate-read selection from a pool of FR pairs held in
    device memory — an 8 Mbp genome, 4000 contigs, 20x coverage (~1.07 M reads), 1% errors; CUDA events
    around the call (median of 3 after a warm-up).  Parity: the same call on a 60-contig pool against the
    oracle (oracle/select.cpp), record by record and byte by byte."""
    import torch
    from gen.pool import make_pool
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    sp = dict(window=150, seed_len=16, seed_stride=4, min_overlap=20, max_mism_pct=4)
    t0 = time.perf_counter()
    pool = make_pool(seed=20211120, genome_len=8_000_000, n_contigs=4000, contig_len=(400, 3000), coverage=20.0,
                     err=0.01, n_rate=1e-4, repeats=20)
    gen_s = time.perf_counter() - t0

    class Dev:
        pass
    dp = Dev()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off"):
        setattr(dp, f, torch.from_numpy(getattr(pool, f)).cuda(dev_i))
    ms = []
    with LocalAssembler(dev_i, stream=stream) as la:
        for i in range(4):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            rec, db = la.select_reads(dp, **sp)
            a1.record(stream)
            a1.synchronize()
            if i:
                ms.append(a0.elapsed_time(a1))
        n_sel = int(rec["sel_end"].size)
        ends_with = int(np.unique(rec["sel_end"]).size)
    med = statistics.median(ms)
    n_reads = 2 * pool.n_pairs
    out = {"api": "la_select_reads (device pool)", "pool_reads": n_reads, "pool_pairs": pool.n_pairs,
           "contigs": pool.n_contigs, "genome_bp": 8_000_000, "coverage": 20.0, "pairs_selected": n_sel,
           "ends_with_reads": ends_with, "ms": med, "value": n_reads / (med / 1e3), "unit": "pool reads/s",
           "params": sp, "gen_s": round(gen_s, 1),
           "note": "NEXT N4, outside the timed step; the synchronous call includes its host round trips for "
                   "buffer sizing (DESIGN.md §10d)"}
    try:
        import oracle
        small = make_pool(seed=20211121, genome_len=60000, n_contigs=60, coverage=25, err=0.015, n_rate=2e-3,
                          repeats=6)
        ref = oracle.select_reads(small.contig_seq, small.contig_off, small.read_seq, small.read_qual,
                                  small.read_off, w=150, s=16, t=4, o=20, mm_pct=4)
        with LocalAssembler(dev_i, stream=stream) as la:
            rec, db = la.select_reads(small, **sp)
            h = db.host()
        bad = sum(int(not np.array_equal(rec[f], ref[f])) for f in ("sel_end", "sel_pair", "sel_flip")) + \
            sum(int(not np.array_equal(h[f], ref[f])) for f in ("end_read_off", "read_off", "read_seq", "read_qual"))
        out["parity"] = {"pairs_checked": int(ref["sel_end"].size), "arrays_differing": bad,
                         "reference": "oracle/select.cpp on a 60-contig, 10k-pair pool"}
    except Exception as ex:   # pragma: no cover
        out["parity"] = {"error": repr(ex)}
    return out


def build_roofline(replay, peaks):
    """Hash-build phase: the build-only replay of the recorded (end, k)
    attempts — stage, prefix, clear, filter + build passes; no link pass, no walk — timed per table
    class with CUDA events.  Shared-memory classes against the shared-memory random-atomic peak, the
    XL class (tables in L2-resident global scratch) against the L2 random RED.ADD peak."""
    ms = statistics.median(r["ms_build"] for r in replay)
    last = replay[-1]
    per = {}
    tot_ins = 0
    for i, n in enumerate(CLASS_NAMES):
        ins = int(last["cls_build_inserts"][i])
        cms = statistics.median(r["cls_build_ms"][i] for r in replay)
        tot_ins += ins
        pk = peaks["l2_gups"] if n.startswith("xl1024") else peaks["smem_gups"]
        ach = ins / (cms / 1e3) / 1e9 if cms > 0 else 0.0
        per[n] = {"inserts": ins, "ms": round(cms, 3), "achieved": ach, "peak": pk,
                  "peak_kind": "l2 RED.ADD" if n.startswith("xl1024") else "smem atomic",
                  "frac": ach / pk if pk else None}
    ach = tot_ins / (ms / 1e3) / 1e9 if ms > 0 else 0.0
    # the denominator of the whole phase: the per-class peaks weighted by the classes' inserts
    w_peak = sum(per[n]["inserts"] * per[n]["peak"] for n in per) / max(tot_ins, 1)
    return {"bound": "smem", "kernel": "table-class kernels in build-only replay (filter + build passes)",
            "achieved": ach, "peak": w_peak, "unit": "G inserts/s", "frac": ach / w_peak if w_peak else None,
            "ms": ms, "inserts": tot_ins, "traffic": None, "classes": per, "peak_src": peaks["smem_src"],
            "note": "per-class fracs use each class's own memory peak; DESIGN.md §7"}


if __name__ == "__main__":
    sys.exit(main())
