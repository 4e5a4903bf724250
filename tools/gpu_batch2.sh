#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for m in 8192 32768 65536 262144; do
  PC_MIN_SLICE_BYTES=$m timeout 600 python tools/sweep.py dl_tensor --ranks 8 --batched | sed "s/^{/{\"min_slice\": $m, /" >> gpurun_out/r02_dlt_batched2.jsonl 2>> gpurun_out/r02_dlt_batched2.err
done
PC_MIN_SLICE_BYTES=65536 timeout 600 python tools/sweep.py dl --ranks 8 --algos direct | sed "s/^{/{\"min_slice\": 65536, /" >> gpurun_out/r02_dlt_batched2.jsonl 2>> gpurun_out/r02_dlt_batched2.err
cat gpurun_out/r02_dlt_batched2.jsonl
