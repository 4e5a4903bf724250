#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_collectives.py -x -q 2>&1 | tail -3 > gpurun_out/r02_coll_pytest.txt
timeout 900 python tools/sweep.py coll --ranks 8,4,2 --max-bytes 1073741824 > gpurun_out/r02_sweep_coll_maxp.jsonl 2> gpurun_out/r02_sweep_coll_maxp.err
cat gpurun_out/r02_coll_pytest.txt
