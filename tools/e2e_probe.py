"""PCIe ceiling vs the host-buffer entry point at a BASELINE config.

  python tools/e2e_probe.py [C3] [reps]      (env BANDLU_HOST_STREAMS / BANDLU_HOST_CHUNK_MB)
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
bpg, n, kl, ku, nrhs, _ = bench.CONFIGS[cfg]
Ah = torch.from_numpy(I.gen_band(n, n, kl, ku, count=bpg)).pin_memory()
Bh = torch.from_numpy(I.gen_rhs(n, nrhs, count=bpg)).pin_memory()
Aw, Bw = torch.empty_like(Ah).pin_memory(), torch.empty_like(Bh).pin_memory()
Ph = torch.zeros((bpg, n), dtype=torch.int32).pin_memory()
Ih = torch.zeros(bpg, dtype=torch.int32).pin_memory()
Ad = torch.empty_like(Ah, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn):
    torch.cuda.synchronize()
    t = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) * 1e3


gb = Ah.numel() * 8 / 1e9
h2d = min(timed(lambda: Ad.copy_(Ah, non_blocking=True)) for _ in range(3))
d2h = min(timed(lambda: Aw.copy_(Ad, non_blocking=True)) for _ in range(3))


def both():
    with torch.cuda.stream(s1):
        Ad.copy_(Ah, non_blocking=True)
    with torch.cuda.stream(s2):
        Aw.copy_(Ad, non_blocking=True)


bi = min(timed(both) for _ in range(3))
e2e = []
for _ in range(reps + 1):
    Aw.copy_(Ah)
    Bw.copy_(Bh)
    e2e.append(timed(lambda: bl.dgbsv_strided_batched_host(n, kl, ku, Aw, Ph, Bw, Ih)))
print(f"{cfg} A={gb:.2f} GB  H2D {gb / h2d * 1e3:.1f} GB/s  D2H {gb / d2h * 1e3:.1f} GB/s  "
      f"both-directions {2 * gb / bi * 1e3:.1f} GB/s  e2e(min of {reps}) {min(e2e[1:]):.2f} ms  "
      f"streams={os.environ.get('BANDLU_HOST_STREAMS', '3')} chunk_mb={os.environ.get('BANDLU_HOST_CHUNK_MB', '64')}")
