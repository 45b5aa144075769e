import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
for (kl, ku, n) in [(2, 32, 7), (2, 32, 40), (2, 2, 12), (4, 4, 13)]:
    A = I.gen_band(n, n, kl, ku, count=1)
    Ao = A.copy(); ipo, io = oracle.dgbtrf(Ao, n, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); P = torch.zeros((1, n), dtype=torch.int32, device='cuda'); inf = torch.zeros(1, dtype=torch.int32, device='cuda')
    bl.dgbtrf_strided_batched(n, n, kl, ku, Ag, P, inf, variant=bl.COLS); torch.cuda.synchronize()
    G = Ag.cpu().numpy()[0]; O = Ao[0]
    print((kl, ku, n), 'ipiv gpu', P.cpu().numpy()[0].tolist(), 'oracle', ipo[0].tolist())
    bad = ~((G == O) | (np.isnan(G) & np.isnan(O)))
    for c, r in np.argwhere(bad)[:12]:
        print('  col', c, 'abrow', r, 'gpu', G[c, r], 'oracle', O[c, r])
