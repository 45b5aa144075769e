"""Compact summary of bench.py JSON lines (files or stdin)."""
import json
import sys

files = sys.argv[1:] or ['-']
for f in files:
    src = sys.stdin if f == '-' else open(f)
    for line in src:
        line = line.strip()
        if not line.startswith('{'):
            continue
        d = json.loads(line)
        if 'unavailable' in d:
            print(f, d)
            continue
        k = d.get('kernels', {})
        r = d.get('roofline', {})
        ks = " ".join(f"{nm}={ms:.4f}ms({gb:.0f}GB/s)" for nm, ms, gb in
                      zip(k.get('launches_per_step', []), k.get('ms', []), k.get('gbs', [])))
        print(f"{d['config'].get('workload', '')[:12]:12s} n_gpus={d.get('n_gpus')} ms/step={d.get('ms_per_step', 0):.4f} "
              f"GF/s={d.get('value', 0):.1f} HBM={d.get('hbm_gbs', 0):.0f}GB/s {ks} frac={r.get('frac', 0):.3f} "
              f"parity={d.get('parity')} e2e={(d.get('e2e') or {}).get('ms_per_step', 0):.1f}ms "
              f"clocks={(d.get('clocks') or {}).get('sm_mhz')} cpu={(d.get('cpu_baseline') or {}).get('value')}")
