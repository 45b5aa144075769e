"""bench.py contract checks that run without a GPU: the reference arm (the CPU
oracle on a bounded sample, task ④) prints one JSON line with the driver's keys,
and the byte / flop accounting used for the roofline matches SURVEY 8(d)'s exact
Σ forms (C3: 212,044 + 135,096 bytes per matrix)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "1", "--warmup", "3",
                        "--config", "C1"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["dtype"] == "f64" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert "workload" in d["config"]


def test_algorithmic_bytes_match_survey_table():
    sys.path.insert(0, ROOT)
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    # SURVEY 8(d), exact sigma forms per matrix (trf + trs)
    assert I.alg_bytes(512, 512, 10, 10, 1) == (212044, 135096)      # C3
    assert I.alg_bytes(64, 64, 2, 2, 1) == (6252, 4760)              # C1
    assert I.alg_bytes(256, 256, 1, 1, 1) == (15316, 13280)          # C2
    assert I.alg_bytes(1024, 1024, 2, 32, 16) == (584892, 564560)    # C4


def test_gpus_flag_self_launches_ranks():
    """`bench.py --gpus 2` without a torchrun environment re-launches itself under
    torch.distributed.run with 2 ranks (127.0.0.1); the reference arm runs on rank 0
    only, so exactly one JSON line comes back, with n_gpus == 2 and the strong-scaling
    global batch."""
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
                        "--warmup", "3", "--config", "C1", "--scaling", "strong"], cwd=ROOT, capture_output=True,
                       text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["config"]["global_batch"] == 100


def test_gpus_flag_must_match_world_size():
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "4", "--steps", "1"], cwd=ROOT, capture_output=True,
                       text=True, timeout=300, env=env)
    assert r.returncode == 2 and "WORLD_SIZE" in r.stderr


def test_torch_generator_matches_numpy_generator():
    """bench.py generates its HBM-sized inputs on the GPU with inputs.gen_band_torch;
    it must reproduce the seeded generator bitwise (checked here on the CPU)."""
    import numpy as np
    sys.path.insert(0, ROOT)
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    for m, n, kl, ku, ldab, first in [(64, 64, 2, 2, None, 0), (30, 20, 3, 2, 12, 7), (512, 512, 10, 10, None, 9999),
                                      (40, 40, 32, 32, None, 2 ** 31 + 5)]:
        a = I.gen_band(m, n, kl, ku, ldab=ldab, count=3, first=first)
        b = I.gen_band_torch(m, n, kl, ku, count=3, first=first, ldab=ldab).numpy()
        assert np.array_equal(np.isnan(a), np.isnan(b)) and np.array_equal(np.nan_to_num(a), np.nan_to_num(b))
    r = I.gen_rhs(50, 3, ldb=53, count=4, first=99)
    t = I.gen_rhs_torch(50, 3, count=4, first=99, ldb=53).numpy()
    assert np.array_equal(np.isnan(r), np.isnan(t)) and np.array_equal(np.nan_to_num(r), np.nan_to_num(t))


def test_bench_parity_checker_catches_a_flipped_bit():
    """bench.py's post-timing parity check (oracle on runs of sampled matrices) reports 0
    mismatches for correct outputs and flags a one-ulp change in one factor entry."""
    import numpy as np
    sys.path.insert(0, ROOT)
    import bench
    import oracle
    from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
    n, kl, ku = 40, 3, 2
    loc = bench.sample_local(300, 24)
    assert 0 in loc and 299 in loc and len(loc) >= 24
    A = np.concatenate([I.gen_band(n, n, kl, ku, count=1, first=i) for i in loc])
    B = np.concatenate([I.gen_rhs(n, 1, count=1, first=i) for i in loc])
    ip, inf = oracle.dgbtrf(A, n, n, kl, ku)
    oracle.dgbtrs(A, ip, B, n, kl, ku)
    assert bench.parity_check(loc, (A, ip, B, inf), n, kl, ku, 1) == 0
    A[3, 5, 5] = np.nextafter(A[3, 5, 5], np.inf)
    assert bench.parity_check(loc, (A, ip, B, inf), n, kl, ku, 1) == 1
    # --trans T: the checker solves A^T X = B with the oracle
    A = np.concatenate([I.gen_band(n, n, kl, ku, count=1, first=i) for i in loc])
    B = np.concatenate([I.gen_rhs(n, 1, count=1, first=i) for i in loc])
    ip, inf = oracle.dgbtrf(A, n, n, kl, ku)
    oracle.dgbtrs(A, ip, B, n, kl, ku, trans="T")
    assert bench.parity_check(loc, (A, ip, B, inf), n, kl, ku, 1, "T") == 0
    assert bench.parity_check(loc, (A, ip, B, inf), n, kl, ku, 1, "N") == len(loc)
