#!/bin/bash
# a6 overlap: the concurrency tests, the whole GPU suite, the DL proxy (fused vs serial vs no-overlap)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_overlap.py -x -q 2>&1 | tail -20 > gpurun_out/r02_overlap_pytest.txt
for f in 0.25 0.5 0.75; do
  PC_OVERLAP_FRAC=$f timeout 600 python tools/dl_bench.py pready,pready_nooverlap,serial,bce_only,allreduce_only 8,4 65536 3 \
    | sed "s/^{/{\"overlap_frac\": $f, /" >> gpurun_out/r02_dl_proxy2.jsonl 2>> gpurun_out/r02_dl_proxy2.err
done
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -30 > gpurun_out/r02_pytest_gpu.txt
tail -3 gpurun_out/r02_overlap_pytest.txt; tail -3 gpurun_out/r02_pytest_gpu.txt; cat gpurun_out/r02_dl_proxy2.jsonl
