import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
kl, ku, n = 2, 32, 7
A = I.gen_band(n, n, kl, ku, count=2)
Ag = torch.from_numpy(A).cuda(); P = torch.zeros((2, n), dtype=torch.int32, device='cuda'); inf = torch.zeros(2, dtype=torch.int32, device='cuda')
bl.dgbtrf_strided_batched(n, n, kl, ku, Ag, P, inf, variant=bl.COLS); torch.cuda.synchronize()
print(P.cpu().numpy())
