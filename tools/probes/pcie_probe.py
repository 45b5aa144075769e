"""Pinned host<->device copy bandwidth on the box (alone and concurrent), and the
host-buffer C-ABI entry point at C3, for the e2e number."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
N = 1 << 30
h = torch.empty(N, dtype=torch.uint8).pin_memory()
h2 = torch.empty(N, dtype=torch.uint8).pin_memory()
d = torch.empty(N, dtype=torch.uint8, device="cuda")
d2 = torch.empty(N, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(fn, reps=3):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps
h2d = t(lambda: d.copy_(h, non_blocking=True))
d2h = t(lambda: h.copy_(d, non_blocking=True))
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
bt = t(both)
print(f"H2D {N/h2d/1e9:.1f} GB/s  D2H {N/d2h/1e9:.1f} GB/s  concurrent: {2*N/bt/1e9:.1f} GB/s total")
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
bpg, n, kl, ku = 10000, 512, 10, 10
Ah = torch.from_numpy(I.gen_band(n, n, kl, ku, count=bpg)).pin_memory()
Bh = torch.from_numpy(I.gen_rhs(n, 1, count=bpg)).pin_memory()
Ph = torch.zeros((bpg, n), dtype=torch.int32).pin_memory(); Ih = torch.zeros(bpg, dtype=torch.int32).pin_memory()
for k in range(4):
    t0 = time.perf_counter()
    bl.dgbsv_strided_batched_host(n, kl, ku, Ah, Ph, Bh, Ih)
    torch.cuda.synchronize()
    print(f"host API call {k}: {1e3*(time.perf_counter()-t0):.1f} ms")
