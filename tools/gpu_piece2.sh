#!/bin/bash
# Interleaved repeats of the C2 step at several D2H piece sizes + the DMA command-shape probe.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/dma_shape_probe.py > gpurun_out/dma_shape_probe.txt 2>&1
for rep in 1 2; do
for p in ${PIECES:-4096 256 512 128}; do
  timeout 600 python bench.py --no-switch --no-migrate --no-c5 --no-cpu --dma-piece-mib $p \
     > gpurun_out/bench_piece${p}_r$rep.json 2> gpurun_out/bench_piece${p}_r$rep.err
done
done
