"""(debug build -DBANDLU_COLS_DEBUG) the incoming entry the owner of column j saw, vs the oracle's
state: A(j+KL, j) after the updates of steps j-KL .. j-1."""
import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_abdelfattahtlad23_b200 as bl
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
kl, ku = 2, 32
for n in (7, 12, 40):
    A = I.gen_band(n, n, kl, ku, count=2)
    B = I.gen_rhs(n, 1, count=2)
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((2, n), dtype=torch.int32, device='cuda'); inf = torch.zeros(2, dtype=torch.int32, device='cuda')
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, inf, phase=bl.TRFS_TWO_LAUNCH | 1)
    torch.cuda.synchronize()
    kv = kl + ku
    orig = [A[0, j, kv + kl] if j + kl < n else 0.0 for j in range(n)]  # A(j+KL, j) original (= incoming value)
    print(n, 'incoming seen', np.round(Bg.cpu().numpy()[0, 0, :n], 4).tolist())
    print(n, 'orig A(j+2,j)', np.round(orig, 4).tolist())
