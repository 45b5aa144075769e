"""Per-opcode histogram from `ncu -i rep --page source --csv --print-source sass`:
executed instructions, stall samples, shared wavefronts, global L1 tag requests
and L2 sectors -- shows which instruction class the kernel's time goes to.

  python tools/sass_hist.py source.csv [top]
"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Source' in r and 'Address' in r)
hdr = rows[hi]
col = {k: hdr.index(k) for k in hdr}


def num(r, k):
    try:
        return float(r[col[k]]) if k in col and r[col[k]] not in ('', '-') else 0.0
    except ValueError:
        return 0.0


keys = ['Instructions Executed', 'Warp Stall Sampling (All Samples)', 'L1 Wavefronts Shared',
        'L1 Wavefronts Shared Ideal', 'L1 Tag Requests Global', 'L2 Theoretical Sectors Global']
agg = collections.defaultdict(lambda: collections.Counter())
static = collections.Counter()
for r in rows[hi + 1:]:
    if len(r) != len(hdr):
        continue
    toks = r[col['Source']].strip().split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith('@') else toks[0]
    base = op.split('.')[0] if not op.startswith(('LDS', 'STS', 'LDG', 'STG')) else op.split('.')[0] + ('.' + op.split('.')[-1] if '.' in op else '')
    for k in keys:
        agg[base][k] += num(r, k)
    static[base] += 1
tot = {k: sum(a[k] for a in agg.values()) or 1 for k in keys}
print('totals:', {k.split(' (')[0]: int(v) for k, v in tot.items()})
print('%-14s %7s %7s %7s %7s %7s %5s' % ('op', 'exec%', 'stall%', 'shwf%', 'gtag%', 'l2sec%', 'stat'))
for op, a in sorted(agg.items(), key=lambda kv: -kv[1][keys[1]])[:int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
    print('%-14s %7.2f %7.2f %7.2f %7.2f %7.2f %5d' % (op, *(100 * a[k] / tot[k] for k in keys[:3]),
                                                     100 * a[keys[4]] / tot[keys[4]], 100 * a[keys[5]] / tot[keys[5]],
                                                     static[op]))
