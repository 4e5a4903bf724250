#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for cfg in "0.5 1" "1.0 1"; do
  set -- $cfg
  PC_OVERLAP_FRAC=$1 PC_OVERLAP_THIN=$2 timeout 300 python tools/dl_bench.py timeline,timeline_serial,allreduce_only,allreduce_bounded 8,4 65536 3 \
    | sed "s/^{/{\"overlap_frac\": $1, \"thin\": $2, /" >> gpurun_out/r02_dl_timeline.jsonl 2>> gpurun_out/r02_dl_timeline.err
done
cat gpurun_out/r02_dl_timeline.jsonl
