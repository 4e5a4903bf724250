#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ll_allreduce.py -x -q 2>&1 | tail -20 > gpurun_out/r02_ll_pytest.txt
for S in 1024 16384 65536 262144; do for a in ll direct rd; do timeout 120 python tools/small_msg_probe.py 8 $S $a; done; done > gpurun_out/r02_ll_probe.txt 2>&1
for S in 1024 65536; do for a in ll direct rd; do timeout 120 python tools/small_msg_probe.py 2 $S $a; done; done >> gpurun_out/r02_ll_probe.txt 2>&1
cat gpurun_out/r02_ll_pytest.txt | tail -5; cat gpurun_out/r02_ll_probe.txt
