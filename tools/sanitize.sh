#!/bin/bash
# compute-sanitizer evidence on the smoke path (C1 swap round trip through gather/scatter kernels)
mkdir -p gpurun_out/sanitizer
for tool in memcheck synccheck racecheck initcheck; do
  timeout 600 compute-sanitizer --tool $tool --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" \
     > gpurun_out/sanitizer/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/$tool.txt
done
