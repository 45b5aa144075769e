#!/usr/bin/env python
"""Benchmark: batched dgbtrf + dgbtrs (the whole hot path) on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl ours|reference]

One STEP = dgbtrf_strided_batched + dgbtrs_strided_batched (two launches of
our sm_100a kernels through the C ABI) over one batch of synthetic band
matrices resident in HBM.  Default workload: BASELINE.json's target config
"batch=10000, n=512, kl=ku=10, nrhs=1 ... at 1/2/4/8 B200" (C3).  Multi-GPU:
one process per GPU (torchrun), each rank factors its own contiguous shard
(10000 matrices per GPU, weak scaling), no collective on the data path; the
time is the max over ranks.  Before every step the pristine A/B are restored
by a device-to-device copy OUTSIDE the timed events; A (1.27 GB per GPU at
C3) is ~10x the 126 MB L2, so inputs are larger than L2.

Reported: value = effective GFLOP/s (nominal, pivot-independent flop count of
SURVEY 8(d)); hbm_gbs = algorithmic bytes (exact SURVEY 8(d) forms) / time;
roofline for the dominant kernel vs MEASURED_PEAKS.json hbm_gbs; e2e through
the host-buffer C-ABI entry point (H2D + D2H inside the timed region);
cpu_baseline = the CPU oracle (test infrastructure) timed on a bounded sample
on the host cores.  --impl reference runs that oracle as the reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "batched dgbtrf+dgbtrs Gflop/s & HBM GB/s (% roofline) vs n,kl,ku at 1/2/4/8 B200"
CONFIGS = {  # name: (batch per GPU, n, kl, ku, nrhs, description)
    "C1": (100, 64, 2, 2, 1, "configs[0]: batch=100, n=64, kl=ku=2, nrhs=1"),
    "C2": (10000, 256, 1, 1, 1, "configs[1]: tridiagonal-like batch=10000, n=256, kl=ku=1, nrhs=1"),
    "C3": (10000, 512, 10, 10, 1, "configs[2]: batch=10000/GPU, n=512, kl=ku=10, nrhs=1 (north_star target)"),
    "C4": (5000, 1024, 2, 32, 16, "configs[3]: batch=5000, n=1024, kl=2, ku=32, nrhs=16"),
    # application-shaped batches (bands synthetic; the paper gives sizes only)
    "XGC": (512, 193, 4, 4, 1, "f4 XGC-like: batch=512, n=193 (P:226-227), kl=ku=4, nrhs=1"),
    "PELE": (10000, 50, 10, 10, 1, "f4 PELE-like: batch=10000, n=50 (P:195-197, 'many <= 50'), kl=ku=10, nrhs=1"),
    # configs[4]: the n sweep, batch per point sized from free HBM (run_sweep)
    "C5": (0, 0, 0, 0, 1, "configs[4]: n sweep 32-2048, (kl,ku) in {(2,3),(10,7),(32,32)}, batch filling HBM"),
}
C5_BANDS = ((2, 3), (10, 7), (32, 32))
C5_NS = (32, 64, 128, 256, 512, 1024, 2048)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


def ncu_traffic(kernel: str, cfg: str):
    """dram bytes per launch for `kernel` at `cfg` from the committed ncu summary, else None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))
        e = d[cfg][kernel]
        return float(e["dram_bytes_read"]) + float(e["dram_bytes_write"])
    except Exception:
        return None


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


def cpu_oracle_rate(n, kl, ku, nrhs, seconds=6.0, sample=None):
    """The CPU oracle (OpenMP over the batch, all host threads) on a bounded
    sample of the workload; returns (matrices/s, sample size, threads, reps)."""
    import oracle
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    if sample is None:
        sample = 1024
    A0 = I.gen_band(n, n, kl, ku, count=sample)
    B0 = I.gen_rhs(n, nrhs, count=sample)
    oracle.build()
    threads = oracle.max_threads()
    best = None
    reps = 0
    t_end = time.perf_counter() + seconds
    while reps < 3 or time.perf_counter() < t_end:
        A, B = A0.copy(), B0.copy()
        t0 = time.perf_counter()
        ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
        oracle.dgbtrs(A, ipiv, B, n, kl, ku)
        dt = time.perf_counter() - t0
        best = dt if best is None else min(best, dt)
        reps += 1
        if reps >= 50:
            break
    return sample / best, sample, threads, reps


def run_sweep(args, rank, world):
    """configs[4]: n = 32..2048 x (kl, ku) in C5_BANDS; per point the
    per-GPU batch fills --fill of free HBM (pristine copy + working copy of A and B),
    weak scaling over ranks.  A seeded block of <= 256 MB is generated per point and
    replicated on the device to the batch (identical per-matrix work; counter-based
    inputs keep every replica bitwise reproducible).  One JSON line: value = total
    nominal flops / total time over the sweep, per-point results under "sweep"."""
    import torch
    import torch.distributed as dist
    import paper_conf_sc_abdelfattahtlad23_b200 as bl
    from paper_conf_sc_abdelfattahtlad23_b200 import dist as bd
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I

    rank, world, dev = bd.init("nccl")
    bl.load()
    st = torch.cuda.current_stream()
    free = torch.cuda.mem_get_info(dev)[0]
    points, tot_flop, tot_ms, tot_bytes = [], 0.0, 0.0, 0.0
    sampler = ClockSampler(torch.cuda.current_device()) if rank == 0 else None
    if sampler:
        sampler.start()
    for kl, ku in C5_BANDS:
        for n in C5_NS:
            ldab = 2 * kl + ku + 1
            per = 2 * 8 * ldab * n + 2 * 8 * n + 4 * n + 4
            bpg = max(1, int(args.fill * free / per))
            gen = max(1, min(bpg, (256 << 20) // (8 * ldab * n)))
            lo, _ = I.shard_range(bpg * world, rank, world)
            blk_a = torch.from_numpy(I.gen_band(n, n, kl, ku, count=gen, first=lo)).to(dev)
            blk_b = torch.from_numpy(I.gen_rhs(n, 1, count=gen, first=lo)).to(dev)
            reps = (bpg + gen - 1) // gen
            A0 = blk_a.repeat(reps, 1, 1)[:bpg].contiguous()
            B0 = blk_b.repeat(reps, 1, 1)[:bpg].contiguous()
            del blk_a, blk_b
            A, B = torch.empty_like(A0), torch.empty_like(B0)
            P = torch.zeros((bpg, n), dtype=torch.int32, device=dev)
            info = torch.zeros(bpg, dtype=torch.int32, device=dev)

            def step(evs=None):
                A.copy_(A0)
                B.copy_(B0)
                if evs is not None:
                    evs[0].record(st)
                bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=1)
                if evs is not None:
                    evs[1].record(st)
                bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=2)
                if evs is not None:
                    evs[2].record(st)

            for _ in range(args.warmup):
                step()
            torch.cuda.synchronize()
            assert int(info.abs().sum()) == 0
            evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            for k in range(args.steps):
                step(evs[k])
            torch.cuda.synchronize()
            trf = sum(e[0].elapsed_time(e[1]) for e in evs) / args.steps
            trs = sum(e[1].elapsed_time(e[2]) for e in evs) / args.steps
            ms, trf, trs = bd.max_over_ranks([trf + trs, trf, trs], dev)
            f_trf, f_trs = I.nominal_flops(n, kl, ku, 1)
            b_trf, b_trs = I.alg_bytes(n, n, kl, ku, 1)
            glob = bpg * world
            points.append({"n": n, "kl": kl, "ku": ku, "batch_per_gpu": bpg, "ms_per_step": ms, "trf_ms": trf,
                           "trs_ms": trs, "gflops": glob * (f_trf + f_trs) / (ms * 1e-3) / 1e9,
                           "hbm_gbs": glob * (b_trf + b_trs) / (ms * 1e-3) / 1e9,
                           "matrices_per_s": glob / (ms * 1e-3), "variant_trf": bl.trf_variant(n, n, kl, ku)})
            tot_flop += glob * (f_trf + f_trs)
            tot_bytes += glob * (b_trf + b_trs)
            tot_ms += ms
            del A0, B0, A, B, P, info
            torch.cuda.empty_cache()
    clocks = sampler.stop() if sampler else None
    if rank == 0:
        peak, peak_kind = peaks()
        best = max(points, key=lambda q: q["hbm_gbs"])
        line = {"metric": METRIC, "value": tot_flop / (tot_ms * 1e-3) / 1e9, "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_ms, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (seeded counter-based U(-1,1) bands, <=256 MB block replicated per point)",
                "config": {"workload": CONFIGS["C5"][5], "fill_of_free_hbm": args.fill, "nrhs": 1,
                           "parallelism": f"batch-shard x{world}", "l2": "inputs larger than L2 (>= 1 GB per point)"},
                "hbm_gbs": tot_bytes / (tot_ms * 1e-3) / 1e9,
                "roofline": {"kernel": "whole step (sweep aggregate)", "bound": "hbm",
                             "achieved": tot_bytes / (tot_ms * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
                             "frac": tot_bytes / (tot_ms * 1e-3) / 1e9 / peak, "peak_kind": peak_kind,
                             "traffic": None, "best_point": {k: best[k] for k in ("n", "kl", "ku", "hbm_gbs")}},
                "e2e": None, "gpu_launches": 2 * args.steps * len(points), "clocks": clocks, "sweep": points}
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C3", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--fill", type=float, default=0.2, help="C5: fraction of free HBM per sweep point")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.config == "C5":
        if args.impl == "reference":
            print(json.dumps({"impl": "reference", "unavailable": "C5 reference arm not run (use a fixed config)"}))
            return
        run_sweep(args, int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")))
        return

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    bpg, n, kl, ku, nrhs, desc = CONFIGS[args.config]
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    b_trf, b_trs = I.alg_bytes(n, n, kl, ku, nrhs)
    fb_trf, fb_trs = I.alg_bytes_fused(n, kl, ku, nrhs)
    f_trf, f_trs = I.nominal_flops(n, kl, ku, nrhs)
    config = {"workload": desc, "batch_per_gpu": bpg, "global_batch": bpg * world, "n": n, "kl": kl, "ku": ku,
              "nrhs": nrhs, "ldab": 2 * kl + ku + 1, "layout": "strided LAPACK band", "parallelism": f"batch-shard x{world}",
              "l2": "inputs larger than L2" if bpg * n * (2 * kl + ku + 1) * 8 > 2 * 126e6
              else "L2 flushed (256 MB write) before every timed step"}

    if args.impl == "reference":
        # Reference arm for this tier = the CPU oracle, rank 0 only.
        if rank != 0:
            return
        rate, sample, threads, reps = cpu_oracle_rate(n, kl, ku, nrhs, seconds=max(3.0, 0.5 * args.steps))
        gflops = rate * (f_trf + f_trs) / 1e9
        line = {"impl": "reference", "metric": METRIC, "value": gflops, "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * bpg * world / rate,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (seeded counter-based U(-1,1) bands)", "config": config,
                "matrices_per_s": rate,
                "cpu_baseline": {"value": gflops, "unit": "GFLOP/s", "cores": threads, "kind": "oracle",
                                 "sample": f"{sample} matrices of the workload, best of {reps} runs"},
                "e2e": {"value": gflops, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line))
        return

    import torch
    import torch.distributed as dist
    import paper_conf_sc_abdelfattahtlad23_b200 as bl
    from paper_conf_sc_abdelfattahtlad23_b200 import dist as bd

    rank, world, dev = bd.init("nccl")  # one process per GPU; NCCL only off the data path
    bl.load()

    # ---- inputs: this rank's shard of the global batch (counter-based generator)
    lo, hi = I.shard_range(bpg * world, rank, world)
    cnt = hi - lo
    A0 = torch.from_numpy(I.gen_band(n, n, kl, ku, count=cnt, first=lo)).to(dev)
    B0 = torch.from_numpy(I.gen_rhs(n, nrhs, count=cnt, first=lo)).to(dev)
    A = torch.empty_like(A0)
    B = torch.empty_like(B0)
    P = torch.zeros((cnt, n), dtype=torch.int32, device=dev)
    info = torch.zeros(cnt, dtype=torch.int32, device=dev)
    flush = None if config["l2"].startswith("inputs larger") else torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    st = torch.cuda.current_stream()

    def step(evs=None):
        A.copy_(A0)
        B.copy_(B0)
        if flush is not None:
            flush.zero_()
        # the hot path: dgbtrf then dgbtrs('N') through dgbtrfs (forward solve
        # fused into the factorization kernel when nrhs == 1); phases 1 / 2
        # are its two launches, timed separately with events in between
        if evs is not None:
            evs[0].record(st)
        bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=1)
        if evs is not None:
            evs[1].record(st)
        bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=2)
        if evs is not None:
            evs[2].record(st)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    assert int(info.abs().sum()) == 0

    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
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
    t_trf = [e[0].elapsed_time(e[1]) for e in evs]
    t_trs = [e[1].elapsed_time(e[2]) for e in evs]
    tot_ms = sum(a + b for a, b in zip(t_trf, t_trs))
    tot_ms, trf_ms, trs_ms = bd.max_over_ranks([tot_ms, sum(t_trf), sum(t_trs)], dev)  # slowest rank
    ms_step = tot_ms / args.steps
    glob = bpg * world
    value = glob * (f_trf + f_trs) / (ms_step * 1e-3) / 1e9
    hbm = glob * (b_trf + b_trs) / (ms_step * 1e-3) / 1e9  # SURVEY 8(d) bytes of trf + trs
    v_trf = bl.trf_variant(n, n, kl, ku)
    fused = nrhs == 1 and v_trf in (bl.WINDOW, bl.ROWS)  # dgbtrfs fuses the forward solve (run_trfs)
    k_trf, k_trs = (fb_trf, fb_trs) if fused else (b_trf, b_trs)  # bytes each launch of THIS path moves
    hbm_moved = glob * (k_trf + k_trs) / (ms_step * 1e-3) / 1e9

    # ---- e2e through the host-buffer C-ABI entry point (H2D + D2H timed)
    e2e_step, h2d, d2h = None, 0, 0
    if args.e2e_steps > 0:
        Ah = torch.from_numpy(I.gen_band(n, n, kl, ku, count=cnt, first=lo)).pin_memory()
        Bh = torch.from_numpy(I.gen_rhs(n, nrhs, count=cnt, first=lo)).pin_memory()
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

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    peak, peak_kind = peaks()
    trf_kernel = {bl.ROWS: "gbtrf_rows_kernel", bl.WINDOW: "gbtrf_window_kernel"}.get(v_trf, "gbtrf_generic_kernel")
    if fused:  # the backward-only launch of dgbtrfs (bandlu.cu launch_trs_bwd)
        trs_kernel = ("gbtrs_rows_kernel" if kl + ku + 1 <= 4 else
                      "gbtrs_bwd_kernel" if kl + ku + 1 <= 32 else "gbtrs_window_kernel")
    else:
        trs_kernel = {bl.WINDOW: "gbtrs_window_kernel", bl.ROWS: "gbtrs_rows_kernel"}.get(
            bl.trs_variant(n, kl, ku, nrhs), "gbtrs_generic_kernel")
    dom = trf_kernel if trf_ms >= trs_ms else trs_kernel
    dom_ms = (trf_ms if trf_ms >= trs_ms else trs_ms) / args.steps
    dom_bytes = cnt * (k_trf if trf_ms >= trs_ms else k_trs)
    achieved = dom_bytes / (dom_ms * 1e-3) / 1e9
    traffic = ncu_traffic(dom, args.config)
    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded counter-based U(-1,1) bands, NaN fill/corners)",
        "config": config,
        "hbm_gbs": hbm, "hbm_frac_of_8TBs": hbm / 8000.0, "hbm_frac_of_measured": hbm / peak,
        "hbm_gbs_moved": hbm_moved,
        "matrices_per_s": glob / (ms_step * 1e-3),
        "kernels": {"gbtrf_ms": trf_ms / args.steps, "gbtrs_ms": trs_ms / args.steps,
                    "gbtrf_gbs": cnt * k_trf / (trf_ms / args.steps * 1e-3) / 1e9,
                    "gbtrs_gbs": cnt * k_trs / (trs_ms / args.steps * 1e-3) / 1e9,
                    "fused_forward_solve": fused,
                    "bytes_per_matrix": {"trf_launch": k_trf, "trs_launch": k_trs, "survey_trf": b_trf,
                                         "survey_trs": b_trs},
                    "variant_trf": bl.trf_variant(n, n, kl, ku), "variant_trs": bl.trs_variant(n, kl, ku, nrhs)},
        "roofline": {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "peak_kind": peak_kind, "traffic": traffic,
                     "alg_bytes_per_launch": dom_bytes},
        "e2e": None if e2e_step is None else {
            "value": glob * (f_trf + f_trs) / (e2e_step * 1e-3) / 1e9, "unit": "GFLOP/s",
            "ms_per_step": e2e_step, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "api": "dgbsv_strided_batched_host (pinned host buffers)"},
        "gpu_launches": 2 * args.steps,
        "clocks": clocks,
    }
    if world == 1 and not args.no_cpu:
        rate, sample, threads, reps = cpu_oracle_rate(n, kl, ku, nrhs)
        line["cpu_baseline"] = {"value": rate * (f_trf + f_trs) / 1e9, "unit": "GFLOP/s", "cores": threads,
                                "kind": "oracle", "matrices_per_s": rate,
                                "sample": f"{sample} matrices of the workload, best of {reps} runs"}
    print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
