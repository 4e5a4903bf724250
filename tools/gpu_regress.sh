#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -3 > gpurun_out/r02_pytest_gpu.txt
timeout 900 python tools/sweep.py allreduce --ranks 8,4,2 --algos auto,direct,ll --partitions 1,16 --max-bytes 1048576 --graph > gpurun_out/r02_sweep_small_graph.jsonl 2>/dev/null
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1
cat gpurun_out/r02_pytest_gpu.txt; tail -1 gpurun_out/r02_smoke.txt
