"""Time dgbtrfs phase 1 (factorization + forward) for experiment builds: time_trfs_lib.py KL KU N BATCH NRHS NAME..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if len(sys.argv) > 6 and sys.argv[6] != "--one":
    for name in sys.argv[6:]:
        r = subprocess.run([sys.executable, __file__, *sys.argv[1:6], "--one", name], capture_output=True, text=True)
        print(name, (r.stdout.strip().splitlines() or [r.stderr[-300:]])[-1])
    sys.exit(0)
kl, ku, n, batch, nrhs = (int(x) for x in sys.argv[1:6])
os.environ["BANDLU_LIB"] = os.path.join(ROOT, "variants_build", f"lib_{sys.argv[7]}.so")
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
B0 = I.gen_rhs_torch(n, nrhs, count=batch, device="cuda")
A, B = torch.empty_like(A0), torch.empty_like(B0)
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
ts = []
for it in range(10):
    A.copy_(A0); B.copy_(B0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=bl.TRFS_TWO_LAUNCH | 1)
    e1.record()
    torch.cuda.synchronize()
    if it >= 3:
        ts.append(e0.elapsed_time(e1))
print(f"trfs phase 1 ({kl},{ku}) n={n} batch={batch} nrhs={nrhs} {bl.trfs_plan(n, kl, ku, nrhs, batch, bl.TRFS_TWO_LAUNCH)['kernels'][0]}: {min(ts):.4f} ms")
