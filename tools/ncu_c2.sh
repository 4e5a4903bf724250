#!/bin/bash
# launch list of C2 epochs (persistent staged producer, block_put INLINE) + full ncu of the producer
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_c2_v4_launches.csv \
  python tools/c2_profile.py 268435456 0 3 persistent > gpurun_out/r02_c2_v4_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vecadd -s 1 -c 2 -o gpurun_out/r02_c2_put_staged -f python tools/c2_profile.py 268435456 0 3 persistent >> gpurun_out/r02_c2_v4_ncu.log 2>&1
tail -3 gpurun_out/r02_c2_v4_ncu.log
