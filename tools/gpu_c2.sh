#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python tools/sweep.py p2p --sizes 16777216,268435456 --grans block --aggs none,1MiB > gpurun_out/r02_c2.jsonl 2> gpurun_out/r02_c2.err
cat gpurun_out/r02_c2.jsonl; tail -3 gpurun_out/r02_c2.err
