"""Small runs of every kernel path, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): every factorization variant compiled for a band, every solve
variant, the fused and two-launch dgbtrfs plans, dgbsv (fused with a singular
matrix, and the two-launch skip path), pointer-array entry points and the
host-buffer path; ragged batches.  Exit code 0 and "sanitize OK" when every result
matched the oracle.

  compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I  # noqa: E402

BANDS = [(0, 0), (0, 3), (1, 1), (2, 2), (2, 3), (3, 0), (3, 2), (4, 4), (10, 7), (10, 10), (2, 32), (32, 32), (5, 6)]
same = lambda a, b: bool(np.all((a == b) | (np.isnan(a) & np.isnan(b))))  # noqa: E731
bad = []


def check(tag, ok):
    if not ok:
        bad.append(tag)


for kl, ku in BANDS:
    n, batch = 40, 19
    A0 = I.gen_band(n, n, kl, ku, count=batch)
    B0 = I.gen_rhs(n, 1, count=batch)
    Ao, Bo = A0.copy(), B0.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    Bt = B0.copy()
    oracle.dgbtrs(Ao, ipo, Bt, n, kl, ku)
    for v in (bl.AUTO, bl.GENERIC, bl.WINDOW, bl.ROWS):
        A = torch.from_numpy(A0.copy()).cuda()
        P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
        info = torch.zeros(batch, dtype=torch.int32, device="cuda")
        try:
            bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info, variant=v)
        except bl.BandLUError:
            continue  # variant not compiled for this band
        torch.cuda.synchronize()
        check(f"trf {kl},{ku} v{v}", same(A.cpu().numpy(), Ao) and np.array_equal(P.cpu().numpy(), ipo))
    for v in (bl.AUTO, bl.GENERIC, bl.WINDOW, bl.ROWS):
        Af = torch.from_numpy(Ao).cuda()
        Pg = torch.from_numpy(ipo).cuda()
        Bg = torch.from_numpy(B0.copy()).cuda()
        try:
            bl.dgbtrs_strided_batched("N", n, kl, ku, Af, Pg, Bg, variant=v)
        except bl.BandLUError:
            continue
        torch.cuda.synchronize()
        check(f"trs {kl},{ku} v{v}", same(Bg.cpu().numpy(), Bt))
    for phase in (0, bl.TRFS_TWO_LAUNCH, bl.TRFS_FUSED):
        A = torch.from_numpy(A0.copy()).cuda()
        B = torch.from_numpy(B0.copy()).cuda()
        P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
        info = torch.zeros(batch, dtype=torch.int32, device="cuda")
        bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=phase)
        torch.cuda.synchronize()
        check(f"trfs {kl},{ku} ph{phase}", same(A.cpu().numpy(), Ao) and same(B.cpu().numpy(), Bt))
    # dgbsv with a singular matrix (B untouched there)
    As = A0.copy()
    kv = kl + ku
    As[3, 7, kl:kv + kl + 1] = np.where(np.isnan(As[3, 7, kl:kv + kl + 1]), np.nan, 0.0)
    Asv, Bsv = As.copy(), B0.copy()
    ips, infs = oracle.dgbsv(Asv, Bsv, n, kl, ku)
    A = torch.from_numpy(As.copy()).cuda()
    B = torch.from_numpy(B0.copy()).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbsv_strided_batched(n, kl, ku, A, P, B, info)
    torch.cuda.synchronize()
    check(f"gbsv {kl},{ku}", same(B.cpu().numpy(), Bsv) and np.array_equal(info.cpu().numpy(), infs))
    # transposed solve
    Bg = torch.from_numpy(B0.copy()).cuda()
    bl.dgbtrs_strided_batched("T", n, kl, ku, torch.from_numpy(Ao).cuda(), torch.from_numpy(ipo).cuda(), Bg)
    Btt = B0.copy()
    oracle.dgbtrs(Ao.copy(), ipo, Btt, n, kl, ku, trans="T")
    torch.cuda.synchronize()
    check(f"trsT {kl},{ku}", same(Bg.cpu().numpy(), Btt))

# ring solves past the truncated edges (n > kv): 'N' one RHS (block solve) and 'T', nrhs 1 and 5
for kl, ku in ((10, 10), (2, 32), (32, 32)):
    n, batch = 150, 7
    A0 = I.gen_band(n, n, kl, ku, count=batch)
    Ao = A0.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    for nrhs in (1, 5):
        B0 = I.gen_rhs(n, nrhs, ldb=n + 1, count=batch)
        for tr in ("N", "T"):
            Bt = B0.copy()
            oracle.dgbtrs(Ao.copy(), ipo, Bt, n, kl, ku, trans=tr)
            Bg = torch.from_numpy(B0.copy()).cuda()
            bl.dgbtrs_strided_batched(tr, n, kl, ku, torch.from_numpy(Ao).cuda(), torch.from_numpy(ipo).cuda(), Bg)
            torch.cuda.synchronize()
            check(f"trs{tr} {kl},{ku} n{n} nrhs{nrhs}", same(Bg.cpu().numpy(), Bt))

# pointer arrays, nrhs 3 (window solve), and the host path
n, kl, ku, nrhs, batch = 33, 10, 10, 3, 9
A0 = I.gen_band(n, n, kl, ku, count=batch)
B0 = I.gen_rhs(n, nrhs, count=batch)
Ao, Bo = A0.copy(), B0.copy()
ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
As = [torch.from_numpy(A0[i].copy()).cuda() for i in range(batch)]
Bs = [torch.from_numpy(B0[i].copy()).cuda() for i in range(batch)]
Ps = [torch.zeros(n, dtype=torch.int32, device="cuda") for _ in range(batch)]
info = torch.zeros(batch, dtype=torch.int32, device="cuda")
bl.dgbsv_batched(n, kl, ku, nrhs, bl.ptr_array(As), 2 * kl + ku + 1, bl.ptr_array(Ps), bl.ptr_array(Bs), n, info, batch)
torch.cuda.synchronize()
check("gbsv ptr", all(same(Bs[i].cpu().numpy(), Bo[i]) for i in range(batch)))
bl.dgbtrf_batched(0, n, kl, ku, bl.ptr_array(As), 2 * kl + ku + 1, torch.zeros(1, dtype=torch.int64, device="cuda"),
                  info, batch)  # quick return: pointer arrays never dereferenced
torch.cuda.synchronize()
At = torch.from_numpy(A0.copy()).pin_memory(); Bt = torch.from_numpy(B0.copy()).pin_memory()
Pt = torch.zeros((batch, n), dtype=torch.int32).pin_memory(); It = torch.zeros(batch, dtype=torch.int32).pin_memory()
bl.dgbsv_strided_batched_host(n, kl, ku, At, Pt, Bt, It)
check("host", same(Bt.numpy(), Bo))
print("sanitize", "OK" if not bad else f"MISMATCH {bad}")
sys.exit(1 if bad else 0)
