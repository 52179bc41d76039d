#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the library's kernels
# (tiny programs, C1, virtual-peer merges, NEXT passes) on one B200.
# usage (from gpurun): bash tools/gpu_sanitize.sh [tag]
TAG=${1:-san}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
CS=/usr/local/cuda/bin/compute-sanitizer
# the subset: every kernel of libdrgpum.so is launched at least once
SEL="tests/test_gpu_parity.py::test_golden_fixtures tests/test_gpu_parity.py::test_tiny_programs \
 tests/test_gpu_parity.py::test_c1_full tests/test_gpu_parity.py::test_c1_host_ingest \
 tests/test_gpu_parity.py::test_empty_and_degenerate tests/test_gpu_parity.py::test_max_range_record \
 tests/test_gpu_parity.py::test_uint32_size_boundary tests/test_gpu_parity.py::test_range_queue_overflow \
 tests/test_gpu_parity.py::test_range_queue_overflow_c1_and_tiny tests/test_gpu_parity.py::test_cuda_graph_replay \
 tests/test_gpu_merge_peers.py::test_owned_state_rules tests/test_gpu_structured.py::test_random_groups_tiny \
 tests/test_gpu_structured.py::test_gramschmidt_polybench_grouped tests/test_gpu_structured.py::test_wide_record_queue_overflow tests/test_gpu_frequency.py::test_sub_calls_and_carried_apis tests/test_gpu_frequency.py::test_c1 \
 tests/test_gpu_merge_peers.py::test_virtual_peers_c1 tests/test_gpu_merge_peers.py::test_virtual_peers_owned_c1 \
 tests/test_gpu_merge_peers.py::test_virtual_peers_owned_tiny_reuse \
 tests/test_gpu_frequency.py::test_tiny tests/test_gpu_frequency.py::test_dependency_chain \
 tests/test_gpu_structured.py::test_tiny tests/test_gpu_structured.py::test_c1 \
 tests/test_gpu_multistream.py::test_c1 tests/test_gpu_small_objects.py"
for tool in memcheck racecheck synccheck; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check no"
  timeout 1500 $CS --tool $tool $extra --print-limit 200 --target-processes all \
      --kernel-name regex=drgpum \
      python -m pytest $SEL -q -p no:cacheprovider > $OUT/$tool.log 2>&1
  echo "$tool rc=$?" | tee -a $OUT/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" $OUT/$tool.log | tail -4 | tee -a $OUT/summary.txt
done
ls -la $OUT
