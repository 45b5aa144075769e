import re, subprocess, sys
log=open('build/ptxas.log').read()
ents=re.split(r"ptxas info    : Compiling entry function '",log)[1:]
for e in ents:
    name=e.split("'")[0]
    if 'Strided' not in name and 'PtrArray' not in name: continue
    if len(sys.argv)>1 and 'PtrArray' in name: continue
    regs=re.search(r"Used (\d+) registers",e); spill=re.search(r"(\d+) bytes spill stores",e)
    dn=subprocess.run(['c++filt',name],capture_output=True,text=True).stdout.strip()
    dn=re.sub(r'bandlu::','',dn)[:100]
    print(regs.group(1) if regs else '?', 'spill',spill.group(1) if spill else '?', dn)
