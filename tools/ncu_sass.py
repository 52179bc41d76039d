"""Dedupe an ncu source CSV (--print-source cuda,sass) by SASS address; print hot regions."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5   # min % of stall samples to print
hdr = None; cur = None; seen = {}
for r in rows:
    if r and r[0] == 'Line No': hdr = r; continue
    if not hdr or not r: continue
    if r[0].isdigit(): cur = r[0] + ':' + r[1].strip()[:45]; continue
    if r[0] == '' and len(r) > 3 and r[2].startswith('0x'):
        a = int(r[2], 16)
        if a in seen: continue
        d = dict(zip(hdr[4:], r[4:]))
        try: seen[a] = (int(d['Instructions Executed'] or 0), int(d['Warp Stall Sampling (All Samples)'] or 0), r[3], cur)
        except ValueError: pass
tot_i = sum(v[0] for v in seen.values()); tot_s = sum(v[1] for v in seen.values())
print(f"unique SASS {len(seen)}, warp-instr {tot_i:,}, stall samples {tot_s:,}")
for a in sorted(seen):
    ex, st, ins, cur = seen[a]
    if st / max(tot_s, 1) * 100 >= thr or ex / max(tot_i, 1) * 100 >= 1.0:
        print(f"{a & 0xffff:5x} ex{ex/tot_i*100:5.2f}% st{st/tot_s*100:5.2f}% {ins[:58]:58s} {cur}")
