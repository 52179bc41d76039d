"""Per-source-line executed warp-instructions and stall samples from an ncu
`--page source --csv --print-source=cuda,sass` export (inlined code is
attributed to the line it came from).  usage: ncu_srclines.py CSV [N]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 50
hdr = None; agg = []
for r in rows:
    if r and r[0] == 'Line No':
        hdr = r; continue
    if hdr and r and r[0].isdigit() and len(r) > 7 and r[7] not in ('-', ''):
        try:
            agg.append((int(r[7]), int(r[4]) if r[4] != '-' else 0, int(r[0]), r[1][:90]))
        except ValueError:
            pass
ti = sum(a[0] for a in agg); ts = sum(a[1] for a in agg)
print(f"total warp-instructions {ti:,}  stall samples {ts:,}")
for ex, st, ln, src in sorted(agg, key=lambda a: -a[0])[:n]:
    print(f"{ln:5d} ex {ex/ti*100:5.1f}% stall {st/max(ts,1)*100:5.1f}% | {src.strip()}")
