"""Histogram of executed SASS opcodes from `ncu --page source --csv` output."""
import csv, collections, sys
rows=list(csv.reader(open(sys.argv[1])))
hdr=rows[1]
si=hdr.index('Source'); ei=hdr.index('Instructions Executed'); wi=hdr.index('Warp Stall Sampling (All Samples)')
ops=collections.Counter(); opsS=collections.Counter(); static=collections.Counter()
tot=0; nstatic=0
for r in rows[2:]:
    if len(r)!=len(hdr) or not r[ei].isdigit(): continue
    toks=r[si].strip().split()
    if not toks: continue
    op=toks[1] if toks[0].startswith('@') else toks[0]
    base=op.split('.')[0]
    n=int(r[ei]); s=int(r[wi] or 0)
    ops[base]+=n; opsS[base]+=s; static[base]+=1; tot+=n; nstatic+=1
print('total executed',tot, 'static', nstatic)
ts=sum(opsS.values()) or 1
for k,v in ops.most_common(int(sys.argv[2]) if len(sys.argv)>2 else 40):
    print('%-10s exec %6.2f%%  stall %6.2f%%  static %d'%(k,100*v/tot,100*opsS[k]/ts,static[k]))
