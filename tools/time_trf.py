"""Time dgbtrf (factorization only) per forced variant: python tools/time_trf.py KL KU N BATCH VARIANT... """
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

kl, ku, n, batch = (int(x) for x in sys.argv[1:5])
names = {"cols": bl.COLS, "rows": bl.ROWS, "tpm": bl.TPM, "window": bl.WINDOW, "generic": bl.GENERIC, "thread": bl.THREAD, "thin": bl.THIN}
A0 = I.gen_band_torch(n, n, kl, ku, count=batch, device="cuda")
A = torch.empty_like(A0)
P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
ref = None
for v in sys.argv[5:]:
    ts = []
    for it in range(8):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info, variant=names[v])
        e1.record()
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(e0.elapsed_time(e1))
    out = (A.clone(), P.clone())
    same = "" if ref is None else (" same" if (torch.equal(torch.nan_to_num(out[0], 7.0), torch.nan_to_num(ref[0], 7.0))
                                               and torch.equal(out[1], ref[1])) else " DIFFERENT")
    ref = ref or out
    print(f"trf ({kl},{ku}) n={n} batch={batch} {v}: {min(ts):.4f} ms{same}")
