"""Compact summary of bench.py JSON lines (files or stdin)."""
import json, sys
files = sys.argv[1:] or ['-']
for f in files:
    src = sys.stdin if f == '-' else open(f)
    for line in src:
        line = line.strip()
        if not line.startswith('{'):
            continue
        d = json.loads(line)
        k = d.get('kernels', {})
        r = d.get('roofline', {})
        print(f"{d['config'].get('workload','')[:12]:12s} n_gpus={d.get('n_gpus')} ms/step={d.get('ms_per_step', 0):.4f} "
              f"GF/s={d.get('value', 0):.1f} HBM={d.get('hbm_gbs', 0):.0f}GB/s "
              f"trf={k.get('gbtrf_ms', 0):.4f}ms({k.get('gbtrf_gbs', 0):.0f}GB/s) trs={k.get('gbtrs_ms', 0):.4f}ms({k.get('gbtrs_gbs', 0):.0f}GB/s) "
              f"frac={r.get('frac', 0):.3f} e2e={(d.get("e2e") or {}).get("ms_per_step", 0):.1f}ms clocks={d.get('clocks', {}).get('sm_mhz')}")
