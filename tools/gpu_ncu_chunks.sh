#!/bin/bash
# ncu metrics of one attribute_kernel launch, chunk shift 13 vs 15 (build/ab/h2, h2s15), on C3 and C5
TAG=${1:-nck}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_red.sum,lts__t_sectors_srcunit_tex_op_red_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_red_lookup_miss.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__pcsamp_warps_issue_stalled_long_scoreboard,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum
cp paper_conf_asplos_linzs23_b200/libdrgpum.so /tmp/lib_default.so
for v in h2 h2s15; do
  cp build/ab/$v/libdrgpum.so paper_conf_asplos_linzs23_b200/libdrgpum.so
  for c in C3 C5; do
    skip=1; [ $c = C5 ] && skip=22
    timeout 600 ncu --metrics $M --clock-control none -k regex:attribute_kernel -s $skip -c 1 --csv \
      python tools/ncu_one.py --config $c > $OUT/m_${v}_$c.csv 2> $OUT/m_${v}_$c.err; echo "$v $c rc=$?"
  done
done
cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so
for f in $OUT/m_*.csv; do echo "== $f"; grep -E "gpu__time|dram__bytes|op_red|hit_rate|inst_exec|issue_active" $f | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'; done
