#!/bin/bash
# session 2 of round 2: memcheck over the new device paths (register Kernel Copy +
# persistent producers, bulk MPI_Wait kernels, cooperative INLINE fold), racecheck over
# the TMA-staged producer's shared-memory ring; then the GPU suite at forced system scope.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
PC_TIMEOUT_MS=120000 timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
 "tests/test_gpu_p2p.py::test_producer_shapes[0-none-3-True]" \
 "tests/test_gpu_p2p.py::test_producer_shapes[0-odd-2-True]" \
 "tests/test_gpu_p2p.py::test_producer_shapes[1-all-1-True]" \
 "tests/test_gpu_p2p.py::test_producer_shapes[0-odd-3-False]" \
 "tests/test_gpu_dl.py::test_dl_proxy_multi_launch[8-6-3000-mixed-0-3-True]" \
 "tests/test_gpu_dl.py::test_dl_proxy_multi_launch[4-13-4099-pready-0-3-True]" > gpurun_out/r02b_memcheck.txt 2>&1
tail -4 gpurun_out/r02b_memcheck.txt
PC_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest -q -x \
 "tests/test_gpu_p2p.py::test_producer_shapes[0-odd-2-True]" > gpurun_out/r02b_racecheck.txt 2>&1
tail -4 gpurun_out/r02b_racecheck.txt
PC_FORCE_SYS_SCOPE=1 timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02b_sys_scope_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/r02b_sys_scope_pytest.log
tail -4 gpurun_out/r02b_sys_scope_pytest.log
