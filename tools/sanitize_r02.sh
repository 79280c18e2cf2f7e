#!/bin/bash
# compute-sanitizer over the round-2 kernel (BULKW) and paths.  memcheck runs the pytest cases;
# racecheck / synccheck cannot start under pytest, so they run tools/sanitize_kernels.py (the same
# test bodies called directly).
mkdir -p gpurun_out/sanitizer_r02
python -c "from paper_conf_sosp_xiang0qyzyzl0025_b200 import build; build.build(force=True)" > /dev/null
AEG_TESTS_NO_REBUILD=1 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -p no:cacheprovider -m gpu \
   "tests/test_gpu_swap.py::test_c1_round_trip_full_images" "tests/test_gpu_edges.py::test_small_shapes_round_trip" \
   "tests/test_gpu_migrate.py::test_local_migrate" "tests/test_gpu_migrate.py::test_local_migrate_under_an_sm_budget" \
   > gpurun_out/sanitizer_r02/memcheck.txt 2>&1
echo "memcheck rc=$?" >> gpurun_out/sanitizer_r02/memcheck.txt
for tool in racecheck synccheck; do
  [ -n "$MEMCHECK_ONLY" ] && break
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_kernels.py \
     > gpurun_out/sanitizer_r02/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer_r02/$tool.txt
done
for f in gpurun_out/sanitizer_r02/*.txt; do echo "== $f"; tail -n 4 $f; done
