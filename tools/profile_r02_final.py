"""Summarise gpurun_out/<tag> of tools/gpu_final_r2.sh / gpu_final_r2b.sh into profiles/<out>.md (run here,
no GPU).  usage: profile_r02_final.py [tag] [out-name]"""
import csv, collections, json, os, subprocess, sys

tag = sys.argv[1] if len(sys.argv) > 1 else "fin1"
out = sys.argv[2] if len(sys.argv) > 2 else "r02_final"
D = f"gpurun_out/{tag}"
L = [f"# Round 2 final capture (`{D}`, `tools/gpu_final_r2.sh` / `tools/gpu_final_r2b.sh`)", ""]
d = json.loads(open(f"{D}/bench.json").read().strip().splitlines()[-1])
keep = {k: d[k] for k in ("value", "unit", "ms_per_step", "phases_ms", "roofline", "parity", "clocks", "e2e",
                          "cpu_baseline", "gpu_launches", "step_exec", "counters", "attribution_paths_tiles")}
keep["config"] = d["config"]
keep["other_configs"] = {c: {k: v.get(k) for k in ("value", "ms_per_step", "phases_ms", "roofline", "parity", "step_exec")}
                         for c, v in d.get("other_configs", {}).items()}
nx = d.get("other_configs", {}).get("C2", {}).get("next")
keep["next_C2"] = nx
L += ["## bench.py (defaults: C5 + other_configs C4, C2)", "", "```json", json.dumps(keep, indent=1), "```", ""]
rows = list(csv.reader(open(f"{D}/launches.csv")))
hdr, agg = None, collections.defaultdict(list)
for r in rows:
    if "Kernel Name" in r: hdr = r; continue
    if hdr and len(r) == len(hdr):
        x = dict(zip(hdr, r))
        if x.get("Metric Name") == "gpu__time_duration.sum":
            v = float(x["Metric Value"]); u = x.get("Metric Unit", "")
            v *= {"usecond": 1e3, "msecond": 1e6, "second": 1e9}.get(u, 1.0)
            agg[x["Kernel Name"].split("(")[0]].append(v)
tot = sum(sum(v) for v in agg.values())
L += ["## Launch list of the default bench (`ncu --metrics gpu__time_duration.sum --clock-control none`, "
      "--steps 2 --warmup 1 --e2e-steps 1; cold-cache, serialised)", "",
      "| kernel | launches | mean us | share of listed time |", "|---|---|---|---|"]
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1]))[:14]:
    L.append(f"| {k} | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {sum(v) / tot * 100:.1f}% |")
L += ["", "(`gen_kernel` is the device trace generator: input generation between chunks, outside the timed events.)", ""]
mets = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors_srcunit_tex_op_red.sum",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
L += ["## ncu --set full captures", "", "| capture | kernel | " + " | ".join(m.split('.')[0] for m in mets) + " |",
      "|---|---|" + "---|" * len(mets)]
traffic = {}
for rep in ("attr_C5", "attr_C2", "fin_C5", "onesweep", "freq_events_kernel", "freq_onesweep_kernel"):
    if not os.path.exists(f"{D}/{rep}.ncu-rep"): continue
    txt = subprocess.run(["ncu", "-i", f"{D}/{rep}.ncu-rep", "--page", "raw", "--csv", "--metrics", ",".join(mets)],
                         capture_output=True, text=True).stdout
    r = list(csv.reader(txt.splitlines()))
    if len(r) < 3: continue
    h, u = r[0], r[1]
    for row in r[2:]:
        x = dict(zip(h, row)); un = dict(zip(h, u))
        L.append(f"| {rep} | {x.get('Kernel Name', '?').split('(')[0][:40]} | " +
                 " | ".join(f"{x.get(m, '')} {un.get(m, '')}".strip() for m in mets) + " |")
        if rep.startswith("attr_"):
            sc = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1}
            b = float(x["dram__bytes_read.sum"]) * sc.get(un["dram__bytes_read.sum"], 1) + \
                float(x["dram__bytes_write.sum"]) * sc.get(un["dram__bytes_write.sum"], 1)
            traffic[rep[5:]] = int(b)
open(f"profiles/{out}.md", "w").write("\n".join(L) + "\n")
t = json.load(open("profiles/traffic.json"))
recs = {"C5": 1 << 30, "C2": 100_000_000}
for c, b in traffic.items():
    t[c] = {"bytes_per_launch": b, "records_per_launch": recs[c],
            "source": f"profiles/{out}.md: ncu --set full of attribute_kernel ({c}, {D}/attr_{c}.ncu-rep): dram read + write per launch"}
json.dump(t, open("profiles/traffic.json", "w"), indent=1)
print(f"profiles/{out}.md", traffic)
