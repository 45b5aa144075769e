"""Multi-process (world_size 2, gloo, CPU) tests of the sharding / timing
logic of the multi-GPU path (pin P11 "sharding invariance").

The GPU kernel is replaced by the CPU oracle here (there is no GPU in CI);
what is under test is the host-side logic bench.py uses: contiguous shards
generated locally from the counter-based generator, no data-path collective,
MAX-over-ranks timing, all-gathered summaries -- and that the per-matrix
results of the sharded run are bitwise identical to the single-process run.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I

N, KL, KU, NRHS, BATCH = 40, 3, 2, 1, 37  # odd batch: unequal shards


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir):
    os.environ.update(RANK=str(rank), WORLD_SIZE=str(world), LOCAL_RANK=str(rank),
                      MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    from paper_conf_sc_abdelfattahtlad23_b200 import dist as bd
    r, w, dev = bd.init("gloo")
    assert (r, w) == (rank, world)
    lo, hi = bd.shard_range(BATCH, r, w)
    A = I.gen_band(N, N, KL, KU, count=hi - lo, first=lo)
    B = I.gen_rhs(N, NRHS, count=hi - lo, first=lo)
    ipiv, info = oracle.dgbsv(A, B, N, KL, KU)
    # fake per-rank "device time": rank-dependent so MAX is observable
    tmax = bd.max_over_ranks([1.0 + r, 10.0 - r], dev)
    summ = bd.gather_summaries([float(hi - lo), float(np.abs(info).sum())], dev)
    np.savez(os.path.join(outdir, f"r{r}.npz"), A=A, B=B, ipiv=ipiv, info=info, lo=lo, hi=hi,
             tmax=np.array(tmax), summ=np.array(summ))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_sharded_run_matches_single_process(tmp_path, world):
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path)), nprocs=world, join=True)
    # single-process reference over the whole batch
    A = I.gen_band(N, N, KL, KU, count=BATCH)
    B = I.gen_rhs(N, NRHS, count=BATCH)
    ipiv, info = oracle.dgbsv(A, B, N, KL, KU)
    covered = np.zeros(BATCH, dtype=bool)
    for r in range(world):
        d = np.load(tmp_path / f"r{r}.npz")
        lo, hi = int(d["lo"]), int(d["hi"])
        assert (lo, hi) == I.shard_range(BATCH, r, world)
        covered[lo:hi] = True
        # bitwise sharding invariance (NaN sentinels included)
        assert np.array_equal(d["A"], A[lo:hi], equal_nan=True)
        assert np.array_equal(d["B"], B[lo:hi], equal_nan=True)
        assert np.array_equal(d["ipiv"], ipiv[lo:hi]) and np.array_equal(d["info"], info[lo:hi])
        # timing is the max over ranks, identical on every rank
        assert list(d["tmax"]) == [float(world), 10.0]
        sizes = [row[0] for row in d["summ"]]
        assert sum(sizes) == BATCH
    assert covered.all()


def test_shard_ranges_partition_the_batch():
    for batch in (1, 7, 10000, 10001):
        for world in (1, 2, 4, 8):
            parts = [I.shard_range(batch, r, world) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == batch
            assert all(parts[i][1] == parts[i + 1][0] for i in range(world - 1))
            sizes = [h - l for l, h in parts]
            assert max(sizes) - min(sizes) <= 1
