"""Summarise an ncu --page source --print-source cuda,sass CSV by source line."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = None; fname = None; agg = []
for r in rows:
    if r and r[0] == 'File Path': fname = r[1].split('/')[-1]
    if r and r[0] == 'Line No': hdr = r; continue
    if hdr and r and r[0].isdigit():
        d = {h: v for h, v in zip(hdr[4:], r[4:])}
        try:
            agg.append((int(d['Instructions Executed'] or 0), int(d['Warp Stall Sampling (All Samples)'] or 0), fname, r[0], r[1][:80], d))
        except ValueError:
            pass
ti = sum(a[0] for a in agg); ts = sum(a[1] for a in agg)
print(f"total warp-instructions {ti:,}  stall samples {ts:,}")
for ex, st, f, ln, src, d in sorted(agg, key=lambda a: -a[1])[:n]:
    top = sorted(((k, int(v)) for k, v in d.items() if k.startswith('stall_') and '(Not' not in k and v.isdigit()), key=lambda kv: -kv[1])[:3]
    print(f"{f}:{ln:>4} ex {ex/ti*100:5.1f}% stall {st/max(ts,1)*100:5.1f}% {top} | {src.strip()}")
