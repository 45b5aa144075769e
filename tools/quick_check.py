"""Quick GPU parity check of one shape (trf+trs) against the oracle; for sanitizer runs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
m, n, kl, ku, batch, nrhs = [int(x) for x in sys.argv[1:7]]
variant = int(sys.argv[7]) if len(sys.argv) > 7 else 0
A = I.gen_band(m, n, kl, ku, count=batch); Ao = A.copy()
ipo, info_o = oracle.dgbtrf(Ao, m, n, kl, ku)
Ag = torch.from_numpy(A).cuda(); P = torch.zeros((batch, max(1, min(m, n))), dtype=torch.int32, device='cuda')
info = torch.zeros(batch, dtype=torch.int32, device='cuda')
bl.dgbtrf_strided_batched(m, n, kl, ku, Ag, P, info, variant=variant); torch.cuda.synchronize()
same = lambda a, b: (a == b) | (np.isnan(a) & np.isnan(b))
ok = same(Ag.cpu().numpy(), Ao)
print('trf factors ok', ok.all(), 'bad', (~ok).sum(), 'ipiv ok', np.array_equal(P.cpu().numpy()[:, :min(m, n)], ipo), 'info ok', np.array_equal(info.cpu().numpy(), info_o))
if m == n:
    B = I.gen_rhs(n, nrhs, count=batch); Bo = B.copy(); oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    Bg = torch.from_numpy(B).cuda()
    bl.dgbtrs_strided_batched('N', n, kl, ku, torch.from_numpy(Ao).cuda(), torch.from_numpy(ipo).cuda(), Bg, variant=variant if variant in (1, 2) else 0)
    torch.cuda.synchronize()
    print('trs ok', same(Bg.cpu().numpy(), Bo).all())
