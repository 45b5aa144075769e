"""dgbtrs('N') / dgbtrfs time for a list of shapes: python tools/time_trsN.py [trs|trfs] KL,KU,N,BATCH ..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

mode = sys.argv[1]
for spec in sys.argv[2:]:
    kl, ku, n, batch = (int(x) for x in spec.split(","))
    A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
    A = A0.clone()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
    B0 = I.gen_rhs_torch(n, 1, count=batch, device="cuda")
    B = torch.empty_like(B0)
    ts = []
    for it in range(6):
        B.copy_(B0)
        if mode == "trfs":
            A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if mode == "trfs":
            bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info)
        else:
            bl.dgbtrs_strided_batched("N", n, kl, ku, A, P, B)
        e1.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    print(f"{mode} ({kl},{kl if False else ku}) n={n} batch={batch}: {min(ts):.3f} ms")
    del A0, A, B, B0, P
    torch.cuda.empty_cache()
