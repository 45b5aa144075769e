import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
m = n = int(sys.argv[1]); kl, ku = int(sys.argv[2]), int(sys.argv[3]); pad = int(sys.argv[4]); variant = int(sys.argv[5])
ldab = 2*kl+ku+1+pad
A = I.gen_band(m, n, kl, ku, ldab=ldab, count=5); Ao = A.copy()
ipo, info_o = oracle.dgbtrf(Ao, m, n, kl, ku)
Ag = torch.from_numpy(A).cuda(); P = torch.zeros((5, n), dtype=torch.int32, device='cuda'); info = torch.zeros(5, dtype=torch.int32, device='cuda')
bl.dgbtrf_strided_batched(m, n, kl, ku, Ag, P, info, variant=variant); torch.cuda.synchronize()
same = lambda a, b: (a == b) | (np.isnan(a) & np.isnan(b))
print(variant, pad, 'ok', same(Ag.cpu().numpy(), Ao).all(), np.array_equal(P.cpu().numpy(), ipo))
