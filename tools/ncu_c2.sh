#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vecadd -s 1 -c 2 -o gpurun_out/r02_c2_vecadd python tools/c2_profile.py 268435456 0 > gpurun_out/r02_ncu_c2.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02_c2_launches.csv python tools/c2_profile.py 268435456 0,1 >> gpurun_out/r02_ncu_c2.log 2>&1
tail -3 gpurun_out/r02_ncu_c2.log
