"""Time dgbtrf (AUTO variant) for one experiment build and compare it bitwise with the reference
build's output saved in /tmp (first call writes it).  usage: time_trf_lib.py KL KU N BATCH NAME"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
kl, ku, n, batch = (int(x) for x in sys.argv[1:5])
name = sys.argv[5]
os.environ["BANDLU_LIB"] = os.path.join(ROOT, "variants_build", f"lib_{name}.so")
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
A = torch.empty_like(A0)
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
ts = []
for it in range(10):
    A.copy_(A0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
    e1.record()
    torch.cuda.synchronize()
    if it >= 3:
        ts.append(e0.elapsed_time(e1))
ref = f"/tmp/trf_ref_{kl}_{ku}_{n}_{batch}.pt"
out = torch.nan_to_num(A, 7.0).cpu(), P.cpu(), info.cpu()
if not os.path.exists(ref):
    torch.save(out, ref)
    same = "ref"
else:
    r = torch.load(ref)
    same = "same" if all(torch.equal(a, b) for a, b in zip(out, r)) else "DIFFERENT"
print(f"trf ({kl},{ku}) n={n} batch={batch}: {min(ts):.4f} ms (median {sorted(ts)[len(ts)//2]:.4f}) {same}")
