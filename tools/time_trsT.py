"""dgbtrs 'N' vs 'T' time after a factorization: python tools/time_trsT.py KL KU N BATCH NRHS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

kl, ku, n, batch, nrhs = (int(x) for x in sys.argv[1:6])
A = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
B0 = I.gen_rhs_torch(n, nrhs, count=batch, device="cuda")
B = torch.empty_like(B0)
b_trf, b_trs = I.alg_bytes(n, n, kl, ku, nrhs)
for tr, var in (("N", bl.AUTO), ("T", bl.AUTO), ("T", bl.GENERIC)):
    ts = []
    for it in range(6):
        B.copy_(B0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        bl.dgbtrs_strided_batched(tr, n, kl, ku, A, P, B, variant=var)
        e1.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    ms = min(ts)
    vn = "generic" if var == bl.GENERIC else "auto"
    print(f"dgbtrs('{tr}', {vn}) ({kl},{ku}) n={n} batch={batch} nrhs={nrhs}: {ms:.3f} ms, {batch * b_trs / ms / 1e6:.0f} GB/s")
