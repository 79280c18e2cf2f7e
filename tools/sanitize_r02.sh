#!/bin/bash
# compute-sanitizer over the round-2 kernel (BULKW) and paths: memcheck + racecheck + synccheck on the
# C1 round trips with every kernel, the small-shape edge cases and the local migrate.
mkdir -p gpurun_out/sanitizer_r02
python -c "from paper_conf_sosp_xiang0qyzyzl0025_b200 import build; build.build(force=True)" > /dev/null
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -m pytest -q -p no:cacheprovider -m gpu \
     "tests/test_gpu_swap.py::test_c1_round_trip_full_images" "tests/test_gpu_edges.py::test_small_shapes_round_trip" \
     "tests/test_gpu_migrate.py::test_local_migrate" "tests/test_gpu_migrate.py::test_local_migrate_under_an_sm_budget" \
     > gpurun_out/sanitizer_r02/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer_r02/$tool.txt
done
tail -3 gpurun_out/sanitizer_r02/*.txt
