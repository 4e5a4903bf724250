#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q 2>&1 | tail -3 > gpurun_out/r02_p2p_pytest.txt
timeout 600 python tools/sweep.py p2p --sizes 1048576,16777216,268435456 --grans block,warp --aggs none,1MiB,all > gpurun_out/r02_c2.jsonl 2> gpurun_out/r02_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_c2_launches2.csv python tools/c2_profile.py 268435456 1 > /dev/null 2>&1
cat gpurun_out/r02_p2p_pytest.txt; tail -3 gpurun_out/r02_c2.err
