#!/bin/bash
# Local hand-off vs layers per launch (AEG_MIGRATE_LOCAL_PACK_MIB), with / without timing events.
mkdir -p gpurun_out
out=gpurun_out/migrate_pack.txt
: > $out
for v in "" "-DAEG_MIGRATE_LOCAL_PACK_MIB=4096" "-DAEG_MIGRATE_LOCAL_PACK_MIB=65536" "-DAEG_MIGRATE_STREAMS=2"; do
  AEG_CXX_EXTRA="$v" python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1 || echo "build failed $v" >> $out
  AEG_CXX_EXTRA="$v" timeout 300 python tools/migrate_pack_probe.py >> $out 2>> gpurun_out/migrate_pack.err
done
python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
timeout 300 python tools/run_leg.py kernel_alone >> $out 2>> gpurun_out/migrate_pack.err
cat $out
# parity of the two-stream variant (migrate tests, race stress, full-size hand-off)
AEG_CXX_EXTRA="-DAEG_MIGRATE_STREAMS=2" timeout 900 python -m pytest tests/test_gpu_migrate.py tests/test_gpu_stress.py \
   tests/test_gpu_c5.py "tests/test_gpu_fullsize.py::test_c3_full_size_handoff" -m gpu -x -q > gpurun_out/migrate2_tests.log 2>&1
tail -3 gpurun_out/migrate2_tests.log
python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
