#!/bin/bash
# BULK ring depth experiment: build with STAGES x PIECE, run the C2 step (no side legs), restore.
mkdir -p gpurun_out
F=paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu
cp $F /tmp/copy.cu.orig
for rep in 1 2; do
for cfg in "6 32768" "7 32768" "3 65536" "12 16384"; do
  set -- $cfg
  cp /tmp/copy.cu.orig $F
  sed -i "s/^constexpr int kBulkStages = 6;/constexpr int kBulkStages = $1;/; s/^constexpr uint32_t kBulkPiece = 32768;/constexpr uint32_t kBulkPiece = $2;/" $F
  python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$1_$2.log 2>&1
  timeout 600 python bench.py --no-switch --no-migrate --no-c5 --no-cpu --no-e2e > gpurun_out/stages_$1_$2_r$rep.json 2> gpurun_out/stages_$1_$2_r$rep.err
done
done
cp /tmp/copy.cu.orig $F
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
