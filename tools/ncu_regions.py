"""Attribute each unique SASS instruction of an ncu source CSV to a code region
by the innermost-function heuristic (the set of attribute.cu lines in its
inline stack), and print executed-instruction and stall-sample totals."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
regions = [tuple(x.split(':')) for x in sys.argv[2].split(',')]   # name:lo-hi ranges (file lines)
per_unit = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
hdr=None; cur=None; fname=None; inst={}
for r in rows:
    if r and r[0]=='File Path': fname=r[1].split('/')[-1]
    if r and r[0]=='Line No': hdr=r; continue
    if not hdr or not r: continue
    if r[0].isdigit(): cur=(fname, int(r[0])); continue
    if r[0]=='' and len(r)>3 and r[2].startswith('0x'):
        a=int(r[2],16); d=dict(zip(hdr[4:],r[4:]))
        e=inst.setdefault(a, [int(d['Instructions Executed'] or 0), int(d['Warp Stall Sampling (All Samples)'] or 0), r[3], set()])
        e[3].add(cur)
def region(lines):
    best=None
    for name,rng in regions:
        lo,hi=map(int,rng.split('-'))
        if any(f=='attribute.cu' and lo<=l<=hi for f,l in lines):
            w=hi-lo
            if best is None or w<best[1]: best=(name,w)
    return best[0] if best else 'other'
ex=collections.Counter(); st=collections.Counter()
for a,(e,s,ins,lines) in inst.items():
    g=region(lines); ex[g]+=e; st[g]+=s
te=sum(ex.values()); ts=sum(st.values())
for g in sorted(ex, key=lambda g:-ex[g]):
    print(f"{g:14s} exec {ex[g]/te*100:5.1f}% ({ex[g]/per_unit:7.1f}/unit)  stall {st[g]/ts*100:5.1f}%")
