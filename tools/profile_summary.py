"""Summarise a gpurun_out/<tag> directory (launch list + ncu --set full captures)
into profiles/<name>.md (tracked).  Run here, without a GPU."""
import csv, collections, json, os, subprocess, sys

tag, out = sys.argv[1], sys.argv[2]
D = f"gpurun_out/{tag}"
lines = [f"# Profile summary ({tag})", ""]
b = json.load(open(f"{D}/bench.json"))
lines += ["## bench.py (C2, N=1)", "", "```", json.dumps({k: b[k] for k in (
    "value", "unit", "ms_per_step", "phases_ms", "roofline", "e2e", "gpu_launches", "clocks",
    "attribution_paths_tiles", "counters")}, indent=1), "```", ""]
rows = list(csv.reader(open(f"{D}/launches.csv"))) if os.path.exists(f"{D}/launches.csv") else []
hdr = None; agg = collections.defaultdict(list)
for r in rows:
    if "Kernel Name" in r: hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            agg[d["Kernel Name"].split("(")[0]].append(float(d["Metric Value"]))
tot = sum(sum(v) for v in agg.values()) or 1.0
if agg:
  lines += ["## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; "
          "bench.py --steps 3 --warmup 3 --e2e-steps 1; cold-cache, serialised: compare shares)", "",
          "| kernel | launches | mean us | share |", "|---|---|---|---|"]
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
  lines.append(f"| {k} | {len(v)} | {sum(v)/len(v)/1e3:.1f} | {sum(v)/tot*100:.1f}% |")
lines.append("")
lines.append("Note: the e2e leg launches the attribution kernel once per 4 Mi-record staging chunk, "
             "so per-launch means mix device-resident (1e8-record) and staged launches.")
lines.append("")
want = ["Duration", "DRAM Throughput", "Memory Throughput", "Executed Instructions",
        "Registers Per Thread", "Achieved Occupancy", "Issue Slots Busy", "L2 Hit Rate",
        "Compute (SM) Throughput", "Grid Size", "Block Size", "Dynamic Shared Memory Per Block"]
for rep in ("attr", "fin"):
    f = f"{D}/{rep}.ncu-rep"
    if not os.path.exists(f):
        continue
    txt = subprocess.run(["ncu", "-i", f, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    lines += [f"## ncu --set full: {rep}", "", "| kernel | metric | unit | value |", "|---|---|---|---|"]
    seen = set()
    for r in csv.reader(txt.splitlines()):
        if len(r) > 14 and r[12] in want and (r[4], r[12]) not in seen:
            seen.add((r[4], r[12]))
            lines.append(f"| {r[4].split('(')[0]} | {r[12]} | {r[13]} | {r[14]} |")
    raw = subprocess.run(["ncu", "-i", f, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    if len(rr) > 2:
        h, units = rr[0], rr[1]
        for row in rr[2:]:
            d = dict(zip(h, row))
            u = dict(zip(h, units))
            name = d.get("Kernel Name", "?").split("(")[0]
            for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"):
                lines.append(f"| {name} | {k} | {u.get(k, '')} | {d.get(k, '')} |")
    lines.append("")
open(out, "w").write("\n".join(lines) + "\n")
print(out)
