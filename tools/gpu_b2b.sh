#!/bin/bash
# back-to-back round trips: enqueue blocking + per-layer timeline, then the swap GPU tests and the bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 400 python tools/b2b_timeline.py --k 4 > gpurun_out/b2b_timeline.json 2> gpurun_out/b2b_timeline.err
timeout 900 python -m pytest tests -m gpu -q \
   -p no:cacheprovider --timeout 400 --timeout-method thread -rA > gpurun_out/gpu_tests_b2b.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gpu_tests_b2b.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
