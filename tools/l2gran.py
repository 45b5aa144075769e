"""Experiment: dgbtrfs at C3 under cudaLimitMaxL2FetchGranularity 0/32/64/128 (device-wide hint).
python tools/l2gran.py"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

rt = ctypes.CDLL("libcudart.so.12")
n, kl, ku, batch = 512, 10, 10, 10000
A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
B0 = I.gen_rhs_torch(n, 1, count=batch, device="cuda")
A, B = A0.clone(), B0.clone()
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for gran in [int(x) for x in (sys.argv[1:] or ["128", "64", "32", "128"])]:
    r = rt.cudaDeviceSetLimit(5, ctypes.c_size_t(gran))
    v = ctypes.c_size_t(0)
    rt.cudaDeviceGetLimit(ctypes.byref(v), 5)
    for phase, nm in ((bl.TRFS_TWO_LAUNCH, "two-launch"),):
        ts = []
        for it in range(8):
            A.copy_(A0); B.copy_(B0); flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=phase)
            e1.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(e0.elapsed_time(e1))
        # the phases separately: 1 = factorization + forward, 2 = backward
        tp = {}
        for ph in (1, 2):
            t2 = []
            for it in range(6):
                if ph == 1:
                    A.copy_(A0); B.copy_(B0)
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=ph | bl.TRFS_TWO_LAUNCH)
                e1.record()
                torch.cuda.synchronize()
                if it >= 2:
                    t2.append(e0.elapsed_time(e1))
            tp[ph] = min(t2)
        print(f"L2 fetch granularity set {gran} (rc {r}, reads back {v.value}): {nm} {min(ts):.4f} ms; "
              f"trf+fwd {tp[1]:.4f} ms, bwd {tp[2]:.4f} ms")
