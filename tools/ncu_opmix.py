"""Instruction mix + stall reasons from an `ncu --page source --csv --print-source sass` dump (first kernel)."""
import csv,sys,collections,re
rows=list(csv.reader(open(sys.argv[1])))
hdr=rows[1]; idx={h:i for i,h in enumerate(hdr)}
stallcols=[h for h in hdr if h.startswith('stall_') and 'Not Issued' not in h]
tot_exec=0; tot_samp=0
byop=collections.Counter(); sampop=collections.Counter(); stalls=collections.Counter()
first=True
for r in rows[2:]:
    if len(r)<len(hdr) or not r[idx['Instructions Executed']].isdigit():
        if r and r[0]=='Kernel Name':
            if not first: break
        continue
    first=False
    src=r[idx['Source']].strip()
    m=re.match(r'(@!?U?P\w+\s+)?([A-Z0-9_]+)',src)
    op=m.group(2) if m else '?'
    ex=int(r[idx['Instructions Executed']]); s=int(r[idx['Warp Stall Sampling (All Samples)']] or 0)
    byop[op]+=ex; sampop[op]+=s; tot_exec+=ex; tot_samp+=s
    for c in stallcols:
        v=r[idx[c]]
        if v and v.replace('.','').isdigit(): stalls[c]+=float(v)
print('total exec',tot_exec,'samples',tot_samp)
for op,c in byop.most_common(int(sys.argv[2]) if len(sys.argv)>2 else 25): print(f'{op:10s} exec {c:10d} {100*c/tot_exec:5.1f}%  stall-samples {100*sampop[op]/max(1,tot_samp):5.1f}%')
ts=sum(stalls.values())
print('stalls:', ', '.join(f'{k[6:]}={100*v/ts:.1f}%' for k,v in stalls.most_common(12)))
