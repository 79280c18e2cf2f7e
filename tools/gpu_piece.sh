#!/bin/bash
# Sub-layer D2H pieces: GPU tests of the swap path, then the C2 step with several piece sizes.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_swap.py tests/test_gpu_stress.py tests/test_gpu_fullsize.py -m gpu -q -p no:cacheprovider \
   --timeout 400 --timeout-method thread -rA > gpurun_out/gpu_tests_piece.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gpu_tests_piece.log
for p in ${PIECES:-4096 128 32 256}; do
  timeout 600 python bench.py --no-switch --no-migrate --no-c5 --no-cpu --dma-piece-mib $p \
     > gpurun_out/bench_piece$p.json 2> gpurun_out/bench_piece$p.err
done
