#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_op_read_hit_rate.pct --clock-control none -k regex:bce_grad -c 40 --csv --log-file gpurun_out/r02_inline_launches.csv python tools/dl_bench.py pready_inline 8 65536 3 > gpurun_out/r02_ncu_inline.log 2>&1
tail -3 gpurun_out/r02_ncu_inline.log
