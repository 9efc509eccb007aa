import re,sys,collections
lines=open('/tmp/all.sass').read().split('\n')
name=sys.argv[1]
start=[i for i,l in enumerate(lines) if 'Function :' in l and name in l][0]
end=[i for i,l in enumerate(lines) if i>start and 'Function :' in l]
end=end[0] if end else len(lines)
ins=[]
for l in lines[start:end]:
    m=re.match(r'\s*/\*([0-9a-f]+)\*/\s+(.*?);',l)
    if m: ins.append(m.group(2))
print(len(ins),'instructions')
DP=('DFMA','DMUL','DADD')
last={}  # reg -> (index, dpcount, op)
dpc=0
hist=collections.Counter(); histI=collections.Counter()
for idx,t in enumerate(ins):
    t=re.sub(r'^@!?U?P\w+\s+','',t)
    op=t.split()[0]
    opb=op.split('.')[0]
    regs=re.findall(r'\bR(\d+)\b',t)
    if not regs: continue
    dst=regs[0]; srcs=regs[1:]
    if opb in DP:
        dists=[]
        for s in srcs:
            for r in (int(s),):
                if r in last and last[r][2] in DP:
                    dists.append((dpc-last[r][1], idx-last[r][0]))
        if dists:
            d=min(dists)
            hist[min(d[0],12)]+=1; histI[min(d[1],30)]+=1
        dpc+=1
    d=int(dst)
    w=2 if opb in DP or op.startswith('LDS.64') or 'MUFU.RCP64' in op or 'MUFU.RSQ64' in op else 1
    for r in range(d,d+w): last[r]=(idx,dpc,opb)
tot=sum(hist.values())
print('DP ops with DP producer:',tot)
print('distance in DP instrs (min over srcs):')
for k in sorted(hist): print(k, hist[k], '%.1f%%'%(100*hist[k]/tot))
