#!/usr/bin/env python
"""Dynamic SASS instruction mix per LDG (and stall share) from `ncu -i X --page source --csv --print-source sass`."""
import csv,sys,collections,re
rows=list(csv.reader(open(sys.argv[1])))
h=rows[1]; ie=h.index("Instructions Executed"); src=h.index("Source"); st=h.index("Warp Stall Sampling (All Samples)")
tot=0; mix=collections.Counter(); stall=collections.Counter(); stot=0
for r in rows[2:]:
    if len(r)<=ie: continue
    try: n=int(r[ie])
    except: continue
    op=r[src].strip().split()
    if not op: continue
    o=op[0]
    if o.startswith('@'): o=op[1]
    o=o.split('.')[0]
    mix[o]+=n; tot+=n
    s=int(r[st] or 0); stall[o]+=s; stot+=s
ldg=mix['LDG']
print("total",tot,"LDG",ldg,"instr/LDG %.2f"%(tot/ldg))
for o,n in mix.most_common(25): print("%-10s %6.2f per LDG   stall share %5.1f%%"%(o,n/ldg,100*stall[o]/stot))
