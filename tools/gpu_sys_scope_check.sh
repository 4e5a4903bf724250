# The GPU suite with every request forced to system-scope ordering
# (PC_FORCE_SYS_SCOPE=1): the fences / acquires / releases the library uses
# between GPUs, exercised on a one-GPU box.
# usage: gpurun --timeout 1500 -- "bash tools/gpu_sys_scope_check.sh"
mkdir -p gpurun_out
PC_FORCE_SYS_SCOPE=1 timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/sys_scope_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/sys_scope_pytest.log
tail -25 gpurun_out/sys_scope_pytest.log
