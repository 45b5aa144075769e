"""One hot-path step (dgbtrf + dgbtrs) at a BASELINE config, for ncu captures.

  python tools/prof_step.py C3 [reps]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
EXTRA = {"C5W": (4000, 512, 32, 32, 1, "C5 (32,32) n=512"), "C5N": (20000, 512, 10, 7, 1, "C5 (10,7) n=512")}
trans = cfg.endswith("T") and cfg[:-1] in bench.CONFIGS  # e.g. C3T: dgbtrf + dgbtrs('T')
bpg, n, kl, ku, nrhs, _ = EXTRA[cfg] if cfg in EXTRA else bench.CONFIGS[cfg[:-1] if trans else cfg]
bpg = int(os.environ.get("PROF_BATCH", bpg))
A0 = I.gen_band_torch(n, n, kl, ku, count=bpg, device='cuda')
B0 = I.gen_rhs_torch(n, nrhs, count=bpg, device='cuda')
A, B = torch.empty_like(A0), torch.empty_like(B0)
P = torch.zeros((bpg, n), dtype=torch.int32, device="cuda")
info = torch.zeros(bpg, dtype=torch.int32, device="cuda")
for _ in range(reps):
    A.copy_(A0)
    B.copy_(B0)
    if os.environ.get("PROF_SEPARATE") or trans:  # plain dgbtrf + dgbtrs launches
        bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
        bl.dgbtrs_strided_batched("T" if trans else "N", n, kl, ku, A, P, B)
    else:  # the bench step: dgbtrfs, every launch of its plan (PROF_TWO: the two-launch plan)
        x = bl.TRFS_TWO_LAUNCH if os.environ.get("PROF_TWO") else 0
        bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=x)
torch.cuda.synchronize()
print("ok", cfg, int(info.abs().sum()))
