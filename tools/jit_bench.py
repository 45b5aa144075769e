"""dgbtrfs throughput (SURVEY 8(d) bytes / step time) for run-time compiled bands next to
their nearest ahead-of-time bands, and the generic kernels' speed on the same bands.

  python tools/jit_bench.py [n] [GB]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
gb = float(sys.argv[2]) if len(sys.argv) > 2 else 1.5
PAIRS = [((5, 6), (4, 4)), ((16, 16), (10, 10)), ((20, 20), (10, 10)), ((0, 32), (2, 32)), ((7, 1), (10, 7))]


def time_trfs(kl, ku, generic=False):
    ldab = 2 * kl + ku + 1
    batch = max(1, int(gb * 1e9 / (8 * ldab * n)))
    A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
    B0 = I.gen_rhs_torch(n, 1, count=batch, device="cuda")
    A, B = torch.empty_like(A0), torch.empty_like(B0)
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    ts = []
    for it in range(6):
        A.copy_(A0)
        B.copy_(B0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if generic:
            bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info, variant=bl.GENERIC)
            bl.dgbtrs_strided_batched("N", n, kl, ku, A, P, B, variant=bl.GENERIC)
        else:
            bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info)
        e1.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    b_trf, b_trs = I.alg_bytes(n, n, kl, ku, 1)
    ms = min(ts)
    return batch, ms, batch * (b_trf + b_trs) / (ms * 1e-3) / 1e9


for jb, cb in PAIRS:
    line = []
    for (kl, ku), tag in ((jb, "jit"), (cb, "aot")):
        batch, ms, gbs = time_trfs(kl, ku)
        line.append(f"{tag} ({kl},{ku}) batch={batch} {ms:.3f} ms {gbs:.0f} GB/s")
    _, msg, gbsg = time_trfs(*jb, generic=True)
    line.append(f"generic ({jb[0]},{jb[1]}) {msg:.3f} ms {gbsg:.0f} GB/s")
    print(" | ".join(line), flush=True)
