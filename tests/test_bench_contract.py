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
