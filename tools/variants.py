"""Build experiment variants of libbandlu.so (only the (1,1)/(10,10) windows)
with different tuning -D flags; run them on the GPU with tools/variants.sh.

usage: python tools/variants.py name=-DFLAG=1,-DFLAG2=3 name2=...
"""
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_abdelfattahtlad23_b200 import _build  # noqa: E402

OUT = os.path.join(ROOT, "variants_build")
os.makedirs(OUT, exist_ok=True)


def one(spec):
    name, flags = spec.split("=", 1)
    flags = [f for f in flags.split(",") if f]
    lib = os.path.join(OUT, f"lib_{name}.so")
    only = [] if name.startswith("F_") else ["-DBANDLU_ONLY_C3"]  # F_*: every band (C4, C5 ...)
    cmd = [_build._nvcc(), *[f for f in _build.NVCC_FLAGS if f != "-v" and f != "-Xptxas"], *only,
           *flags, _build.SRC, "-o", lib]
    r = subprocess.run(cmd, capture_output=True, text=True)
    return name, r.returncode, r.stderr[-800:]


with ThreadPoolExecutor(max_workers=4) as ex:
    for name, rc, err in ex.map(one, sys.argv[1:]):
        print(name, "OK" if rc == 0 else "FAIL\n" + err)
with open(os.path.join(OUT, "list.txt"), "w") as f:
    for spec in sys.argv[1:]:
        f.write(spec.split("=", 1)[0] + "\n")
