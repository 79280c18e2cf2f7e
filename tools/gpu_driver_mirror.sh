#!/bin/bash
# Mirror of the driver's round-end GPU steps: pytest -m gpu, smoke(), bench (N=1) and the reference arm.
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
t0=$(date +%s)
timeout 2400 python -m pytest tests -x -q -m gpu -rA > gpurun_out/gpu_tests.log 2>&1; echo "pytest rc=$? $(( $(date +%s)-t0 ))s" >> gpurun_out/gpu_tests.log
t0=$(date +%s)
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$? $(( $(date +%s)-t0 ))s" >> gpurun_out/smoke.log
t0=$(date +%s)
timeout 600 python bench.py --impl reference --gpus 1 --steps ${REF_STEPS:-20} --warmup ${REF_WARMUP:-5} > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$? $(( $(date +%s)-t0 ))s" >> gpurun_out/bench_ref.err
t0=$(date +%s)
timeout 3000 python bench.py --gpus 1 --steps ${STEPS:-20} --warmup ${WARMUP:-5} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$? $(( $(date +%s)-t0 ))s" >> gpurun_out/bench.err
for f in gpurun_out/gpu_tests.log gpurun_out/smoke.log gpurun_out/bench_ref.err gpurun_out/bench.err; do tail -n 3 $f; done
