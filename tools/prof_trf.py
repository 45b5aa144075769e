"""One dgbtrf launch with a forced variant (ncu captures): python tools/prof_trf.py KL KU N BATCH VARIANT"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

kl, ku, n, batch = (int(x) for x in sys.argv[1:5])
v = {"rows": bl.ROWS, "tpm": bl.TPM, "window": bl.WINDOW, "generic": bl.GENERIC}[sys.argv[5]]
A = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info, variant=v)
torch.cuda.synchronize()
print("ok")
