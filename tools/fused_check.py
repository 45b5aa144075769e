"""GPU dgbtrfs (fused factor + forward solve, then backward solve) vs the oracle's dgbtrf + dgbtrs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
n, kl, ku, batch = [int(x) for x in sys.argv[1:5]]
A = I.gen_band(n, n, kl, ku, count=batch); B = I.gen_rhs(n, 1, count=batch)
Ao, Bo = A.copy(), B.copy()
ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku); oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
Ag, Bg = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
P = torch.zeros((batch, n), dtype=torch.int32, device='cuda'); info = torch.zeros(batch, dtype=torch.int32, device='cuda')
bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, info); torch.cuda.synchronize()
same = lambda a, b: (a == b) | (np.isnan(a) & np.isnan(b))
print('fused', n, kl, ku, 'A', same(Ag.cpu().numpy(), Ao).all(), 'ipiv', np.array_equal(P.cpu().numpy(), ipo),
      'info', np.array_equal(info.cpu().numpy(), info_o), 'B', same(Bg.cpu().numpy(), Bo).all())
