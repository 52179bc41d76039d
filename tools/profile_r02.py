import csv, subprocess, json
mets=["gpu__time_duration.sum","dram__bytes_read.sum","dram__bytes_write.sum","lts__t_sectors_srcunit_tex_op_red.sum",
      "smsp__inst_executed.sum","smsp__issue_active.avg.pct_of_peak_sustained_active","sm__warps_active.avg.pct_of_peak_sustained_active",
      "lts__t_sector_hit_rate.pct","gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
recs={"C2":100_000_000,"C3":1_000_000_000,"C4":4_000_000_000,"C5":1<<30}
L=["# Round 2: ncu captures of the attribution kernel on every benchmarked config\n",
   "Source: `gpurun_out/r2b` (`tools/gpu_ncu_r2.sh`): `ncu --set full --clock-control none --import-source on -k regex:attribute_kernel` "
   "on `tools/ncu_one.py --config CX` (bench.py's `Workload` step; device-generated records; the second step's launch; C5: "
   "chunk 8 of the 15 2^30-record launches of a step).  One B200, 1965 MHz.  Per launch.  Build: round-2 HEAD before the union-scratch / sparse-reset change.\n",
   "| config | records / launch | duration | DRAM read | DRAM write | traffic / (16 B x records) | RED sectors at L2 | RED sectors / record | warp-inst / record | issue active | achieved occupancy | L2 hit | DRAM throughput |",
   "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
out={}; traffic={}
for c in recs:
    txt=subprocess.run(["ncu","-i",f"gpurun_out/r2b/attr_{c}.ncu-rep","--page","raw","--csv","--metrics",",".join(mets)],capture_output=True,text=True).stdout
    r=list(csv.reader(txt.splitlines())); h=r[0]; u=r[1]; v=r[2]
    out[c]={k:(x,un) for k,un,x in zip(h,u,v) if k in mets}
def num(c,k):
    x,u=out[c][k]; x=float(x)
    return x*{"Gbyte":1e9,"Mbyte":1e6,"Kbyte":1e3,"byte":1,"msecond":1e-3,"usecond":1e-6,"nsecond":1e-9,"ms":1e-3,"us":1e-6}.get(u,1)
for c,n in recs.items():
    d=num(c,"gpu__time_duration.sum"); rd=num(c,"dram__bytes_read.sum"); wr=num(c,"dram__bytes_write.sum")
    red=num(c,"lts__t_sectors_srcunit_tex_op_red.sum"); ins=num(c,"smsp__inst_executed.sum")
    traffic[c]=int(rd+wr)
    g=lambda k: float(out[c][k][0])
    L.append(f"| {c} | {n:.3g} | {d*1e3:.3f} ms | {rd/1e9:.3f} GB | {wr/1e6:.1f} MB | {(rd+wr)/(16*n):.3f} | {red/1e6:.1f} M | {red/n:.3f} | {ins/n:.2f} | "
             f"{g('smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f}% | {g('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f}% | "
             f"{g('lts__t_sector_hit_rate.pct'):.1f}% | {g('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed'):.1f}% |")
L.append("""
Reading: every config's DRAM traffic is within a few % of the 16 B/record stream (no wasted re-reads).  The
kernel is issue-bound: issue slots 61-65% busy at 35-37% achieved occupancy (3 blocks x 8 warps, 80
registers, 72.6 KB of shared memory per block); top stall reasons `wait` (fixed-latency dependencies),
then `long_scoreboard` / `short_scoreboard` / `not_selected`; the L2 RED traffic (0.14-0.26 sectors per
record) is the second cost.  C5 tiles by path (bench r2a): 45.6% affine union, 0.8% affine per-record
words, 53.0% in-object / tile fast path, 0.6% slow.  Per-line breakdown: `ncu -i gpurun_out/r2b/attr_C5.ncu-rep
--page source --csv --print-source=cuda,sass` (C5 top lines: the affine-tier check 5.6% of instructions,
the in-object tier's per-record element ranges, the ring's lane-0 fetch bookkeeping).

## C5 launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, bench.py --steps 2 --warmup 1, cold-cache, serialised)

| kernel | launches | mean | note |
|---|---|---|---|
| tracegen gen_kernel | 91 | 4.51 ms | input generation, outside the timed events |
| attribute_kernel | 282 | 1.09 ms | 15 x 3.2 ms launches per step + the e2e leg's 4 Mi-record staged launches |
| object_finalize_kernel | 9 | 1.57 ms | one warp per object, 10^6 objects |
| tile_reduce_kernel | 9 | 0.67 ms | |
| reset_kernel | 10 | 0.28 ms | |
| range_expand_kernel | 282 | 3.1 us | |
| group_reduce_kernel | 9 | 44 us | |

Share of a C5 step's library kernel time (15 x 3.23 + 1.57 + 0.67 + 0.28 + 0.04 ms): attribution 94%, finalize 4.5%, reset 0.5%
-- consistent with bench.py's in-context phases (attribute 48.45 ms, finalize 2.37 ms, reset 0.29 ms of 51.2 ms).
""")
open("profiles/r02_ncu_attribution_c2_c5.md","w").write("\n".join(L)+"\n")
json.dump({c:{"bytes_per_launch":traffic[c],"records_per_launch":recs[c],
              "source":f"profiles/r02_ncu_attribution_c2_c5.md: ncu --set full of attribute_kernel ({c}, gpurun_out/r2b/attr_{c}.ncu-rep): dram__bytes_read.sum + dram__bytes_write.sum per launch"} for c in traffic},
          open("profiles/traffic.json","w"), indent=1)
