#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:direct_engine_group -s 2 -c 1 \
  -o gpurun_out/r02_thin_engine python tools/dl_bench.py allreduce_bounded 8 65536 3 > gpurun_out/r02_ncu_thin.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:direct_engine_group -s 2 -c 1 \
  -o gpurun_out/r02_fat_engine python tools/dl_bench.py allreduce_only 8 65536 3 > gpurun_out/r02_ncu_fat.log 2>&1
tail -3 gpurun_out/r02_ncu_thin.log gpurun_out/r02_ncu_fat.log
