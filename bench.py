#!/usr/bin/env python
"""Benchmark: batched dgbtrf + dgbtrs (the whole hot path) on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3]
                  [--scaling weak|strong] [--impl ours|reference]

One STEP = the hot path over one batch of synthetic band matrices resident
in HBM: dgbtrf followed by dgbtrs('N') through the C ABI entry point
dgbtrfs_strided_batched (the factorization kernel applies the forward
substitution on the fly for nrhs == 1, then the backward solve runs -- in the
same kernel or a second launch, whichever the library picks for the shape;
every launch is one of our sm_100a kernels).  Default workload: BASELINE.json
"batch=10000, n=512, kl=ku=10, nrhs=1 ... at 1/2/4/8 B200" (C3).

Multi-GPU: one process per GPU.  `--gpus N` without a torchrun environment
re-launches itself under torch.distributed.run (N ranks, 127.0.0.1).  Every
rank generates and factors its own contiguous shard (counter-based generator,
no scatter, no collective on the data path); NCCL carries only the barrier
and the MAX-over-ranks device time.  --scaling weak (default, the task's
"shard the units" rule): the config's batch per GPU; --scaling strong: the
config's batch is the GLOBAL batch, split by inputs.shard_range.

Timing: W untimed warm-up steps, then K steps timed with CUDA events on the
launching stream.  Before every step the pristine A/B are restored by a
device-to-device copy OUTSIDE the events; C2-C4 inputs are far larger than L2,
C1 flushes L2 (256 MB write) before each step.  After the timed region a
sample of the last step's outputs (first/last/random matrices of every rank's
shard) is compared bitwise with the CPU oracle ("parity"); a mismatch exits 1.

Reported: value = effective GFLOP/s (nominal, pivot-independent flop count of
SURVEY 8(d)); hbm_gbs = SURVEY 8(d) algorithmic bytes / time; roofline of the
dominant kernel vs MEASURED_PEAKS.json; e2e through the host-buffer C-ABI entry
point dgbsv_strided_batched_host (H2D + D2H inside the timed region);
cpu_baseline = the CPU oracle (test infrastructure) on a bounded sample, all
host threads and 1 thread.  --impl reference runs that oracle as the
reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "batched dgbtrf+dgbtrs Gflop/s & HBM GB/s (% roofline) vs n,kl,ku at 1/2/4/8 B200"
CONFIGS = {  # name: (batch per GPU (weak) / global (strong), n, kl, ku, nrhs, description)
    "C1": (100, 64, 2, 2, 1, "configs[0]: batch=100, n=64, kl=ku=2, nrhs=1"),
    "C2": (10000, 256, 1, 1, 1, "configs[1]: tridiagonal-like batch=10000, n=256, kl=ku=1, nrhs=1"),
    "C3": (10000, 512, 10, 10, 1, "configs[2]: batch=10000, n=512, kl=ku=10, nrhs=1 (north_star target)"),
    "C4": (5000, 1024, 2, 32, 16, "configs[3]: batch=5000, n=1024, kl=2, ku=32, nrhs=16"),
    # application-shaped batches (bands synthetic; the paper gives sizes only)
    "XGC": (512, 193, 4, 4, 1, "f4 XGC-like: batch=512, n=193 (P:226-227), kl=ku=4, nrhs=1"),
    "PELE": (10000, 50, 10, 10, 1, "f4 PELE-like: batch=10000, n=50 (P:195-197, 'many <= 50'), kl=ku=10, nrhs=1"),
    # configs[4]: the n sweep, batch per point sized from free HBM (run_sweep)
    "C5": (0, 0, 0, 0, 1, "configs[4]: n sweep 32-2048, (kl,ku) in {(2,3),(10,7),(32,32)}, batch filling HBM"),
}
C5_BANDS = ((2, 3), (10, 7), (32, 32))
C5_NS = (32, 64) + tuple(range(128, 2049, 128))  # 18 points per band


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic(kernel: str, cfg: str):
    """dram bytes per launch for `kernel` at `cfg` from the committed ncu summary, else None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))
        e = d[cfg][kernel]
        return float(e["dram_bytes_read"]) + float(e["dram_bytes_write"])
    except Exception:
        return None


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.12)
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except Exception:
            self.proc.kill()
            out = ""
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0])); smax.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------- CPU legs
# The oracle (oracle/, test infrastructure) runs ONLY here: the cpu_baseline /
# reference-arm timing and the post-timing parity check of a sample of the
# GPU's outputs.  Neither is inside a timed GPU region.

def cpu_oracle_rate(n, kl, ku, nrhs, seconds=6.0, sample=1024, threads=0, trans="N"):
    """The CPU oracle (OpenMP over the batch; threads=0: all host threads) on a
    bounded sample of the workload.  Returns a dict with matrices/s (best and
    median over the repetitions), the sample size, threads used and reps."""
    import oracle
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    A0 = I.gen_band(n, n, kl, ku, count=sample)
    B0 = I.gen_rhs(n, nrhs, count=sample)
    oracle.build()
    if threads <= 0:  # every host core (explicit: an earlier call may have changed the OpenMP default)
        threads = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    used = threads
    times = []
    t_end = time.perf_counter() + seconds
    while len(times) < 3 or (time.perf_counter() < t_end and len(times) < 50):
        A, B = A0.copy(), B0.copy()
        t0 = time.perf_counter()
        ipiv, info = oracle.dgbtrf(A, n, n, kl, ku, nthreads=threads)
        oracle.dgbtrs(A, ipiv, B, n, kl, ku, trans=trans, nthreads=threads)
        times.append(time.perf_counter() - t0)
    return {"best": sample / min(times), "median": sample / statistics.median(times), "sample": sample,
            "threads": used, "reps": len(times)}


def cpu_baseline_entry(n, kl, ku, nrhs, flops_per_matrix, seconds=6.0, trans="N"):
    allt = cpu_oracle_rate(n, kl, ku, nrhs, seconds=seconds, trans=trans)
    one = cpu_oracle_rate(n, kl, ku, nrhs, seconds=max(2.0, seconds / 3), sample=max(16, allt["sample"] // 8),
                          threads=1, trans=trans)
    g = lambda r: r * flops_per_matrix / 1e9  # noqa: E731
    return {"value": g(allt["best"]), "unit": "GFLOP/s", "cores": allt["threads"], "kind": "oracle",
            "matrices_per_s": allt["best"], "median_gflops": g(allt["median"]),
            "one_thread": {"value": g(one["best"]), "median": g(one["median"]), "matrices_per_s": one["best"],
                           "sample": one["sample"], "reps": one["reps"]},
            "cpu_model": cpu_model(), "nproc": os.cpu_count(),
            "sample": f"{allt['sample']} matrices of the workload (all threads, best of {allt['reps']}); "
                      f"{one['sample']} matrices on 1 thread (best of {one['reps']})"}


def parity_check(idx_global, outs, n, kl, ku, nrhs, trans="N"):
    """Bitwise comparison of GPU outputs (A, ipiv, B, info per sampled matrix)
    with the oracle recomputed from the same seeded inputs (runs of consecutive
    matrices regenerated and factored as one OpenMP batch).  Returns mismatches."""
    import oracle
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    Ag, Pg, Bg, Ig = outs
    same = lambda a, b: np.all((a == b) | (np.isnan(a) & np.isnan(b)), axis=tuple(range(1, a.ndim)))  # noqa: E731
    bad, k = 0, 0
    idx = [int(i) for i in idx_global]
    while k < len(idx):
        e = k
        while e + 1 < len(idx) and idx[e + 1] == idx[e] + 1:
            e += 1
        cnt = e - k + 1
        Ao = I.gen_band(n, n, kl, ku, count=cnt, first=idx[k])
        Bo = I.gen_rhs(n, nrhs, count=cnt, first=idx[k])
        ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
        oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku, trans=trans)
        sl = slice(k, e + 1)
        ok = ((Ig[sl] == info_o) & np.all(Pg[sl] == ipo, axis=1) & same(Ag[sl], Ao) & same(Bg[sl], Bo))
        bad += int(np.sum(~ok))
        k = e + 1
    return bad


def sample_local(cnt, k, seed=11):
    """Local indices to verify: the first and last matrix of the shard and at least
    min(k, cnt) more, in non-overlapping runs of consecutive matrices at random run
    slots (runs keep the oracle batched)."""
    if cnt <= 0:
        return []
    rng = np.random.default_rng(seed)
    run = max(8, k // 16)
    slots = max(1, cnt // run)
    take = min(slots, -(-k // run))
    s = {0, cnt - 1}
    for st in rng.choice(slots, size=take, replace=False):
        s.update(int(st) * run + o for o in range(run) if int(st) * run + o < cnt)
    return sorted(s)


# --------------------------------------------------------------- launcher
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch_distributed(nproc: int, argv: list[str]) -> int:
    """Run this script under torch.distributed.run with `nproc` ranks (one per GPU)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__), *argv]
    return subprocess.call(cmd)


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C3", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    ap.add_argument("--batch", type=int, default=0, help="override the config's batch (per GPU weak / global strong)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--parity-sample", type=int, default=24, help="random matrices per rank checked vs the oracle")
    ap.add_argument("--fill", type=float, default=0.3, help="C5: fraction of free HBM per sweep point")
    ap.add_argument("--plan", default="auto", choices=["auto", "two", "fused", "thin"],
                    help="dgbtrfs plan: the library's choice, the two-launch plan (factorization + forward, then "
                         "backward), or the fused single-launch kernel")
    ap.add_argument("--trans", default="N", choices=["N", "T"],
                    help="T: the step is dgbtrf then dgbtrs('T') (A^T X = B, SURVEY 8(f) f2), two launches")
    ap.add_argument("--c5-ns", default="", help="C5: comma-separated n list (default 32,64,128..2048 step 128)")
    args = ap.parse_args(argv)
    args.warmup = max(args.warmup, 3)
    return args


# --------------------------------------------------------------- GPU arm
def run_config(args):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_abdelfattahtlad23_b200 as bl
    from paper_conf_sc_abdelfattahtlad23_b200 import dist as bd
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I

    bcfg, n, kl, ku, nrhs, desc = CONFIGS[args.config]
    if args.batch > 0:
        bcfg = args.batch
    rank, world, dev = bd.init("nccl")  # one process per GPU; NCCL only off the data path
    bl.load()
    glob = bcfg * world if args.scaling == "weak" else bcfg
    lo, hi = I.shard_range(glob, rank, world)
    cnt = hi - lo
    ldab = 2 * kl + ku + 1
    b_trf, b_trs = I.alg_bytes(n, n, kl, ku, nrhs)
    f_trf, f_trs = I.nominal_flops(n, kl, ku, nrhs)
    xph = {"auto": 0, "two": bl.TRFS_TWO_LAUNCH, "fused": bl.TRFS_FUSED, "thin": bl.TRFS_THIN}[args.plan]
    plan = bl.trfs_plan(n, kl, ku, nrhs, cnt, xph)  # the kernels one dgbtrfs call launches
    if args.trans == "T":  # dgbtrf (no forward fusion: nrhs 2 never fuses it) + dgbtrs('T')
        plan = {"kernels": [bl.trfs_plan(n, kl, ku, 2, cnt, 0)["kernels"][0], "gbtrs_t_kernel"],
                "bytes": ["trf", "trs"], "fused": False}
    per_launch_bytes = [I.alg_bytes_kind(n, kl, ku, nrhs, k) for k in plan["bytes"]]
    big = cnt * n * ldab * 8 > 2 * 126e6
    if args.trans == "T":
        desc += "; solve A^T X = B (dgbtrs 'T')"
    config = {"workload": desc, "global_batch": glob, "batch_per_gpu": cnt, "n": n, "kl": kl, "ku": ku,
              "nrhs": nrhs, "ldab": ldab, "layout": "strided LAPACK band (minimal ldab)",
              "parallelism": f"batch-shard x{world} ({args.scaling} scaling)",
              "l2": "inputs larger than L2" if big else "L2 flushed (256 MB write) before every timed step"}

    A0 = I.gen_band_torch(n, n, kl, ku, count=cnt, first=lo, device=dev)
    B0 = I.gen_rhs_torch(n, nrhs, count=cnt, first=lo, device=dev)
    A, B = torch.empty_like(A0), torch.empty_like(B0)
    P = torch.zeros((cnt, n), dtype=torch.int32, device=dev)
    info = torch.zeros(cnt, dtype=torch.int32, device=dev)
    flush = None if big else torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    st = torch.cuda.current_stream()
    nph = len(plan["kernels"])

    def step(evs=None):
        A.copy_(A0)
        B.copy_(B0)
        if flush is not None:
            flush.zero_()
        # the hot path: dgbtrf then dgbtrs('N') through dgbtrfs; its launches
        # (phase 1, phase 2 when there is a second one) are timed separately
        if evs is not None:
            evs[0].record(st)
        if args.trans == "T":
            bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
            if evs is not None:
                evs[1].record(st)
            bl.dgbtrs_strided_batched("T", n, kl, ku, A, P, B)
            if evs is not None:
                evs[2].record(st)
            return
        for ph in range(1, nph + 1):
            bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=(ph if nph > 1 else 0) | xph)
            if evs is not None:
                evs[ph].record(st)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(nph + 1)] for _ in range(args.steps)]
    sampler = ClockSampler(torch.cuda.current_device()) if rank == 0 else None
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if sampler:
        sampler.start()
    for k in range(args.steps):
        step(evs[k])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop() if sampler else None
    per_ph = [sum(e[p].elapsed_time(e[p + 1]) for e in evs) for p in range(nph)]
    tot = bd.max_over_ranks([sum(per_ph)] + per_ph, dev)  # slowest rank
    ms_step = tot[0] / args.steps
    ph_ms = [t / args.steps for t in tot[1:]]

    # ---- parity of the timed outputs: a sample of the last step, every rank
    loc = sample_local(cnt, args.parity_sample)
    sel = torch.tensor(loc, device=dev)
    outs = tuple(t.index_select(0, sel).cpu().numpy() for t in (A, P, B, info))
    ninfo = int((info != 0).sum())
    bad = parity_check([lo + i for i in loc], outs, n, kl, ku, nrhs, args.trans)
    summ = bd.gather_summaries([len(loc), bad, ninfo], dev)
    checked, mism, ninfo = (int(sum(s[k] for s in summ)) for k in range(3))

    # ---- e2e through the host-buffer C-ABI entry point (H2D + D2H timed)
    e2e = None
    if args.e2e_steps > 0 and args.trans == "N":  # the host-buffer entry point is dgbsv ('N')
        Ah = A0.cpu().pin_memory()
        Bh = B0.cpu().pin_memory()
        Ahw, Bhw = torch.empty_like(Ah).pin_memory(), torch.empty_like(Bh).pin_memory()
        Ph = torch.zeros((cnt, n), dtype=torch.int32).pin_memory()
        Ih = torch.zeros(cnt, dtype=torch.int32).pin_memory()
        e2e_ms = []
        for k in range(args.e2e_steps + 1):
            Ahw.copy_(Ah); Bhw.copy_(Bh)
            if world > 1:
                dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            bl.dgbsv_strided_batched_host(n, kl, ku, Ahw, Ph, Bhw, Ih)  # synchronous
            e1.record(st)
            torch.cuda.synchronize()
            if k > 0:
                e2e_ms.append(e0.elapsed_time(e1))
        e2e_step = bd.max_over_ranks([sum(e2e_ms) / len(e2e_ms)], dev)[0]
        h2d = Ah.numel() * 8 + Bh.numel() * 8
        d2h = Ah.numel() * 8 + Ph.numel() * 4 + Bh.numel() * 8 + Ih.numel() * 4
        e2e = {"value": glob * (f_trf + f_trs) / (e2e_step * 1e-3) / 1e9, "unit": "GFLOP/s",
               "ms_per_step": e2e_step, "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world,
               "api": "dgbsv_strided_batched_host (pinned host buffers, chunked H2D/kernels/D2H pipeline)"}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0 if mism == 0 else 1

    peak, peak_kind = peaks()
    dom = int(np.argmax(ph_ms))
    dom_ms = ph_ms[dom]
    dom_bytes = cnt * per_launch_bytes[dom]
    achieved = dom_bytes / (dom_ms * 1e-3) / 1e9
    value = glob * (f_trf + f_trs) / (ms_step * 1e-3) / 1e9
    hbm = glob * (b_trf + b_trs) / (ms_step * 1e-3) / 1e9  # SURVEY 8(d) bytes of trf + trs
    moved = glob * sum(per_launch_bytes) / (ms_step * 1e-3) / 1e9
    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": args.scaling,
        "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded counter-based U(-1,1) bands generated on the GPU, NaN fill/corners)",
        "config": config,
        "hbm_gbs": hbm, "hbm_frac_of_8TBs": hbm / 8000.0, "hbm_frac_of_measured": hbm / peak,
        "hbm_gbs_path_bytes": moved,
        "matrices_per_s": glob / (ms_step * 1e-3),
        "kernels": {"launches_per_step": plan["kernels"], "ms": ph_ms,
                    "gbs": [cnt * b / (t * 1e-3) / 1e9 for b, t in zip(per_launch_bytes, ph_ms)],
                    "alg_bytes_per_matrix": per_launch_bytes, "survey_bytes_per_matrix": [b_trf, b_trs],
                    "fused": plan["fused"]},
        "roofline": {"kernel": plan["kernels"][dom], "bound": "hbm", "achieved": achieved, "peak": peak,
                     "unit": "GB/s", "frac": achieved / peak, "peak_kind": peak_kind,
                     "traffic": ncu_traffic(plan["kernels"][dom], args.config),
                     "alg_bytes_per_launch": dom_bytes},
        "parity": {"checked": checked, "mismatches": mism, "info_nonzero": ninfo,
                   "what": "first/last/random matrices of every shard, last timed step, bitwise vs the CPU oracle"},
        "e2e": e2e,
        "gpu_launches": nph * args.steps,
        "clocks": clocks,
    }
    if world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline_entry(n, kl, ku, nrhs, f_trf + f_trs, trans=args.trans)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0 if mism == 0 else 1


def run_sweep(args):
    """configs[4]: n in C5_NS x (kl, ku) in C5_BANDS; per point the
    per-GPU batch fills --fill of free HBM (pristine + working copy of A and B),
    generated on the GPU (no replicated blocks), weak scaling over ranks.  One JSON
    line: value = total nominal flops / total time over the sweep; per-point results
    (with a parity sample each) under "sweep"."""
    import torch
    import torch.distributed as dist
    import paper_conf_sc_abdelfattahtlad23_b200 as bl
    from paper_conf_sc_abdelfattahtlad23_b200 import dist as bd
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I

    rank, world, dev = bd.init("nccl")
    bl.load()
    ns = tuple(int(x) for x in args.c5_ns.split(",")) if args.c5_ns else C5_NS
    st = torch.cuda.current_stream()
    free = torch.cuda.mem_get_info(dev)[0]
    points, tot_flop, tot_ms, tot_bytes, checked, mism, launches = [], 0.0, 0.0, 0.0, 0, 0, 0
    sampler = ClockSampler(torch.cuda.current_device()) if rank == 0 else None
    if sampler:
        sampler.start()
    for kl, ku in C5_BANDS:
        for n in ns:
            ldab = 2 * kl + ku + 1
            per = 2 * 8 * ldab * n + 2 * 8 * n + 4 * n + 4
            bpg = max(1, int(args.fill * free / per))
            lo, _ = I.shard_range(bpg * world, rank, world)
            A0 = I.gen_band_torch(n, n, kl, ku, count=bpg, first=lo, device=dev)
            B0 = I.gen_rhs_torch(n, 1, count=bpg, first=lo, device=dev)
            A, B = torch.empty_like(A0), torch.empty_like(B0)
            P = torch.zeros((bpg, n), dtype=torch.int32, device=dev)
            info = torch.zeros(bpg, dtype=torch.int32, device=dev)
            xph = {"auto": 0, "two": bl.TRFS_TWO_LAUNCH, "fused": bl.TRFS_FUSED, "thin": bl.TRFS_THIN}[args.plan]
            plan = bl.trfs_plan(n, kl, ku, 1, bpg, xph)
            nph = len(plan["kernels"])

            def step(evs=None):
                A.copy_(A0)
                B.copy_(B0)
                if evs is not None:
                    evs[0].record(st)
                for ph in range(1, nph + 1):
                    bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=(ph if nph > 1 else 0) | xph)
                    if evs is not None:
                        evs[ph].record(st)

            for _ in range(args.warmup):
                step()
            torch.cuda.synchronize()
            evs = [[torch.cuda.Event(enable_timing=True) for _ in range(nph + 1)] for _ in range(args.steps)]
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            for k in range(args.steps):
                step(evs[k])
            torch.cuda.synchronize()
            per_ph = [sum(e[p].elapsed_time(e[p + 1]) for e in evs) / args.steps for p in range(nph)]
            r = bd.max_over_ranks([sum(per_ph)] + per_ph, dev)
            ms = r[0]
            loc = sample_local(bpg, max(4, args.parity_sample // 4))
            sel = torch.tensor(loc, device=dev)
            outs = tuple(t.index_select(0, sel).cpu().numpy() for t in (A, P, B, info))
            bad = parity_check([lo + i for i in loc], outs, n, kl, ku, 1)
            f_trf, f_trs = I.nominal_flops(n, kl, ku, 1)
            b_trf, b_trs = I.alg_bytes(n, n, kl, ku, 1)
            glob = bpg * world
            points.append({"n": n, "kl": kl, "ku": ku, "batch_per_gpu": bpg, "ms_per_step": ms, "kernel_ms": r[1:],
                           "kernels": plan["kernels"], "gflops": glob * (f_trf + f_trs) / (ms * 1e-3) / 1e9,
                           "hbm_gbs": glob * (b_trf + b_trs) / (ms * 1e-3) / 1e9,
                           "matrices_per_s": glob / (ms * 1e-3), "parity_checked": len(loc), "parity_bad": bad})
            tot_flop += glob * (f_trf + f_trs)
            tot_bytes += glob * (b_trf + b_trs)
            tot_ms += ms
            checked += len(loc)
            mism += bad
            launches += nph * args.steps
            del A0, B0, A, B, P, info
            torch.cuda.empty_cache()
    clocks = sampler.stop() if sampler else None
    summ = bd.gather_summaries([checked, mism], dev)
    checked, mism = int(sum(s[0] for s in summ)), int(sum(s[1] for s in summ))
    if rank == 0:
        peak, peak_kind = peaks()
        best = max(points, key=lambda q: q["hbm_gbs"])
        agg = tot_bytes / (tot_ms * 1e-3) / 1e9
        line = {"metric": METRIC, "value": tot_flop / (tot_ms * 1e-3) / 1e9, "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_ms, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (seeded counter-based U(-1,1) bands generated on the GPU per point)",
                "config": {"workload": CONFIGS["C5"][5], "fill_of_free_hbm": args.fill, "nrhs": 1, "ns": list(ns),
                           "parallelism": f"batch-shard x{world}", "l2": "inputs larger than L2 (>= 1 GB per point)"},
                "hbm_gbs": agg,
                "roofline": {"kernel": "whole step (sweep aggregate)", "bound": "hbm", "achieved": agg,
                             "peak": peak, "unit": "GB/s", "frac": agg / peak, "peak_kind": peak_kind,
                             "traffic": None, "best_point": {k: best[k] for k in ("n", "kl", "ku", "hbm_gbs")}},
                "parity": {"checked": checked, "mismatches": mism},
                "e2e": None, "gpu_launches": launches, "clocks": clocks, "sweep": points}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0 if mism == 0 else 1


def run_reference(args):
    """Reference arm for this tier = the CPU oracle (rank 0 only), on this arm's
    config / metric / unit, each step a bounded sample of the workload."""
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if rank != 0:
        return 0
    if args.config == "C5":
        print(json.dumps({"impl": "reference", "unavailable": "C5 reference arm not run (use a fixed config)"}))
        return 0
    bcfg, n, kl, ku, nrhs, desc = CONFIGS[args.config]
    if args.batch > 0:
        bcfg = args.batch
    glob = bcfg * world if args.scaling == "weak" else bcfg
    f_trf, f_trs = I.nominal_flops(n, kl, ku, nrhs)
    r = cpu_oracle_rate(n, kl, ku, nrhs, seconds=max(3.0, 0.5 * args.steps), trans=args.trans)
    gflops = r["best"] * (f_trf + f_trs) / 1e9
    if args.trans == "T":
        desc += "; solve A^T X = B (dgbtrs 'T')"
    config = {"workload": desc, "global_batch": glob, "n": n, "kl": kl, "ku": ku, "nrhs": nrhs,
              "ldab": 2 * kl + ku + 1, "parallelism": f"batch-shard x{world} ({args.scaling} scaling)"}
    line = {"impl": "reference", "metric": METRIC, "value": gflops, "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * glob / r["best"],
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded counter-based U(-1,1) bands)", "config": config,
            "matrices_per_s": r["best"],
            "cpu_baseline": {"value": gflops, "unit": "GFLOP/s", "cores": r["threads"], "kind": "oracle",
                             "cpu_model": cpu_model(), "median": r["median"] * (f_trf + f_trs) / 1e9,
                             "sample": f"{r['sample']} matrices of the workload per step, best of {r['reps']} runs"},
            "e2e": {"value": gflops, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return relaunch_distributed(args.gpus, argv)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        return 2
    if args.impl == "reference":
        return run_reference(args)
    if args.config == "C5":
        return run_sweep(args)
    return run_config(args)


if __name__ == "__main__":
    sys.exit(main())
