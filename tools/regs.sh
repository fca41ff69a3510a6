#!/bin/bash
# registers / spills per flux kernel instantiation (ptxas -v)
cd "$(dirname "$0")/.."
python -m paper_conf_ipps_heislersdms24_b200.build --force -v 2>&1 | python -c "
import sys,re,subprocess
cur=None
for l in sys.stdin:
    m=re.search(r\"Compiling entry function '(\S+)'\",l)
    if m: cur=subprocess.run(['c++filt',m.group(1)],capture_output=True,text=True).stdout.strip().replace('bte::','').replace('(FluxParams)','')
    m=re.search(r'(\d+) bytes spill stores',l)
    if m and cur: sp=m.group(1)
    m=re.search(r'Used (\d+) registers',l)
    if m and cur and 'flux' in cur: print('%-45s regs %3s spill %s'%(cur,m.group(1),sp))
"
