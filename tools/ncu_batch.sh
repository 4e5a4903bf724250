#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"epoch_batch|direct_engine_batch" -c 12 --csv --log-file gpurun_out/r02_batch_launches.csv python tools/sweep.py dl_tensor --ranks 8 --batched > gpurun_out/r02_ncu_batch.log 2>&1
tail -3 gpurun_out/r02_ncu_batch.log
