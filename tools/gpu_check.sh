# One gpurun call: full GPU suite, smoke, bench (own arm + reference arm); logs under gpurun_out/.
# usage: gpurun --timeout 2700 -- "bash tools/gpu_check.sh"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r01_check_gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01_check_pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/r01_check_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r01_check_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/r01_check_smoke.log
timeout 600 python bench.py > gpurun_out/r01_check_bench.log 2>&1; echo "bench exit $?" >> gpurun_out/r01_check_bench.log
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r01_check_bench_ref.log 2>&1; echo "ref exit $?" >> gpurun_out/r01_check_bench_ref.log
tail -3 gpurun_out/r01_check_pytest_gpu.log; tail -2 gpurun_out/r01_check_smoke.log; tail -c 600 gpurun_out/r01_check_bench.log
