#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/c2_floor tools/c2_floor.cu
timeout 120 /tmp/c2_floor 256 > gpurun_out/r02_c2_floor3.jsonl 2>&1
timeout 600 python tools/sweep.py p2p --sizes 268435456 --grans block_put --aggs none --persistent > gpurun_out/r02_c2_v5_pers.jsonl 2>&1
cat gpurun_out/r02_c2_floor3.jsonl; cut -c1-200 gpurun_out/r02_c2_v5_pers.jsonl
