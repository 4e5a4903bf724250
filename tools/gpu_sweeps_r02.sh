#!/bin/bash
# round-2 parity-gated sweeps (C5 allreduce, C2 p2p, NEXT-3 collectives)
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1800 python tools/sweep.py allreduce --ranks 8,4,2 --algos direct,direct_push,ring,rd --partitions 1,16,64 --max-bytes 1073741824 > gpurun_out/r02_sweep_c5.jsonl 2> gpurun_out/r02_sweep_c5.err
timeout 900 python tools/sweep.py p2p --sizes 65536,1048576,16777216,268435456 > gpurun_out/r02_sweep_c2_full.jsonl 2> gpurun_out/r02_sweep_c2_full.err
timeout 900 python tools/sweep.py coll --ranks 8,4 --max-bytes 1073741824 > gpurun_out/r02_sweep_coll_full.jsonl 2> gpurun_out/r02_sweep_coll_full.err
wc -l gpurun_out/r02_sweep_*.jsonl; tail -2 gpurun_out/r02_sweep_c5.err gpurun_out/r02_sweep_c2_full.err gpurun_out/r02_sweep_coll_full.err
