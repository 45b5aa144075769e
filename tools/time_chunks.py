"""dgbtrfs (phase 0, what the bench step calls) time and a checksum of the outputs, under the
BANDLU_TRFS_CHUNKS setting of this process: python tools/time_chunks.py [batch n kl ku]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

batch, n, kl, ku = (int(x) for x in (sys.argv[1:5] if len(sys.argv) > 4 else (10000, 512, 10, 10)))
A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
B0 = I.gen_rhs_torch(n, 1, count=batch, device="cuda")
A, B = torch.empty_like(A0), torch.empty_like(B0)
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
ts = []
for it in range(12):
    A.copy_(A0); B.copy_(B0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info)
    e1.record()
    torch.cuda.synchronize()
    if it >= 3:
        ts.append(e0.elapsed_time(e1))
h = (A.view(torch.int64).sum().item(), B.view(torch.int64).sum().item(), P.sum().item(), info.sum().item())
ts.sort()
print(f"chunks={os.environ.get('BANDLU_TRFS_CHUNKS', 'default')} batch={batch} n={n} ({kl},{ku}): "
      f"min {ts[0]:.4f} med {ts[len(ts) // 2]:.4f} ms  checksum {h}")
