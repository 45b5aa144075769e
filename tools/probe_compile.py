"""Compile selected kernel instantiations to a cubin and print regs / SASS size.
usage: python tools/probe_compile.py trf|trs KL,KU [KL,KU ...]"""
import subprocess, sys, re
kind=sys.argv[1]; pairs=[tuple(map(int,a.split(','))) for a in sys.argv[2:]]
hdr={'trf':'gbtrf_window.cuh','trs':'gbtrs_window.cuh'}[kind]
lines=['#include "%s"'%hdr,'using namespace bandlu;','void* probes[] = {']
for kl,ku in pairs:
    if kind=='trf':
        lines.append('(void*)&gbtrf_window_kernel<%d,%d,true,Strided<double>,Strided<int>,Strided<double>>,'%(kl,ku))
    else:
        lines.append('(void*)&gbtrs_window_kernel<%d,%d,Strided<const double>,Strided<const int>,Strided<double>>,'%(kl,ku))
lines.append('};')
open('/tmp/_bandlu_probe.cu','w').write('\n'.join(lines)+'\n')
r=subprocess.run('nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --fmad=false -Xptxas -v -I paper_conf_sc_abdelfattahtlad23_b200/csrc -cubin -o /tmp/probe.cubin /tmp/_bandlu_probe.cu',shell=True,capture_output=True,text=True)
for l in r.stderr.splitlines():
    if 'error' in l or 'Used' in l or 'spill' in l or 'Compiling' in l: print(l[:200])
s=subprocess.run('cuobjdump -sass /tmp/probe.cubin',shell=True,capture_output=True,text=True).stdout
cur=None; cnt={}
for l in s.splitlines():
    m=re.search(r'Function : (\S+)',l)
    if m: cur=m.group(1); cnt[cur]=0
    elif cur and re.search(r'/\*[0-9a-f]{4,}\*/',l): cnt[cur]+=1
for k,v in cnt.items(): print(v, k[:80])
open('/tmp/probe.sass','w').write(s)
