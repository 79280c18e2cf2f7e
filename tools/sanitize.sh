#!/bin/bash
# compute-sanitizer evidence on the smoke path (C1 swap round trip through gather/scatter kernels)
mkdir -p gpurun_out/sanitizer
for tool in memcheck synccheck racecheck initcheck; do
  timeout 600 compute-sanitizer --tool $tool --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" \
     > gpurun_out/sanitizer/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/$tool.txt
done
# memcheck over the sub-layer (D2H piece) swap tests: gate kernel, two swap-outs, chained swap-ins
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_swap.py -m gpu -q \
   -p no:cacheprovider -k "piece or chained" > gpurun_out/sanitizer/memcheck_pieces.txt 2>&1
echo "memcheck_pieces rc=$?" >> gpurun_out/sanitizer/memcheck_pieces.txt
