#!/bin/bash
# Local hand-off vs layers per launch (AEG_MIGRATE_LOCAL_PACK_MIB; default 4096), with / without
# timing events.  (The two-kernel-stream variant measured in profiles/r02/migrate_pack.txt gave no
# gain and was removed from the library.)
mkdir -p gpurun_out
out=gpurun_out/migrate_pack.txt
: > $out
for v in "-DAEG_MIGRATE_LOCAL_PACK_MIB=512" "" "-DAEG_MIGRATE_LOCAL_PACK_MIB=65536"; do
  AEG_CXX_EXTRA="$v" python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1 || echo "build failed $v" >> $out
  AEG_CXX_EXTRA="$v" timeout 300 python tools/migrate_pack_probe.py >> $out 2>> gpurun_out/migrate_pack.err
done
python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
timeout 300 python tools/run_leg.py kernel_alone >> $out 2>> gpurun_out/migrate_pack.err
cat $out
