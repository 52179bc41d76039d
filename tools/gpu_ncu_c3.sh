#!/bin/bash
# C3 with 8192- vs 32768-record chunks: SM activity and stall reasons of one attribute_kernel launch
TAG=${1:-nc3}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
M=gpu__time_duration.sum,sm__cycles_active.avg,sm__cycles_active.max,sm__cycles_active.min,sm__cycles_elapsed.avg,smsp__warps_active.avg.per_cycle_active,smsp__inst_executed.sum,smsp__average_warp_latency_issue_stalled_long_scoreboard,smsp__pcsamp_warps_issue_stalled_long_scoreboard,smsp__pcsamp_warps_issue_stalled_wait,smsp__pcsamp_warps_issue_stalled_short_scoreboard,smsp__pcsamp_warps_issue_stalled_lg_throttle,smsp__pcsamp_warps_issue_stalled_membar,smsp__pcsamp_warps_issue_stalled_drain,smsp__pcsamp_warps_issue_stalled_barrier,smsp__pcsamp_warps_issue_stalled_mio_throttle,smsp__pcsamp_sample_count,lts__t_sectors_srcunit_tex_op_atom.sum,l1tex__t_set_conflicts_pipe_lsu_mem_global_op_red.sum
cp paper_conf_asplos_linzs23_b200/libdrgpum.so /tmp/lib_default.so
for v in s13 s15; do
  cp build/ab/$v/libdrgpum.so paper_conf_asplos_linzs23_b200/libdrgpum.so
  timeout 600 ncu --metrics $M --clock-control none -k regex:attribute_kernel -s 1 -c 1 --csv \
      python tools/ncu_one.py --config C3 > $OUT/m_$v.csv 2> $OUT/m_$v.err; echo "$v rc=$?"
done
cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so
for f in $OUT/m_*.csv; do echo "== $f"; grep -v "^==" $f | awk -F'","' 'NR>1{print $(NF-2), $(NF-1), $NF}'; done
