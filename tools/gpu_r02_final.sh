#!/bin/bash
# round-2 final measurement set (session 2): full GPU suite, smoke, bench N=1, reference arm,
# ncu launch list of the bench command, ncu --set full of the dominant kernel and of the C2 put producer
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -5 > gpurun_out/r02c_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02c_smoke.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02c_bench_n1.json 2> gpurun_out/r02c_bench_n1.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r02c_bench_ref_n1.json 2> gpurun_out/r02c_bench_ref_n1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02c_launches_bench_n1.csv \
  python bench.py --steps 2 --warmup 1 --no-c1 --no-jacobi --no-latency --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:direct_engine_group -s 3 -c 1 \
  -o gpurun_out/r02c_direct_engine_group -f python bench.py --steps 2 --warmup 3 --no-c1 --no-jacobi --no-latency --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vecadd -s 1 -c 2 \
  -o gpurun_out/r02c_c2_put_persistent -f python tools/c2_profile.py 268435456 0 3 persistent > /dev/null 2>&1
tail -3 gpurun_out/r02c_pytest_gpu.txt; tail -1 gpurun_out/r02c_smoke.txt; cut -c1-400 gpurun_out/r02c_bench_n1.json; cut -c1-200 gpurun_out/r02c_bench_ref_n1.json; tail -3 gpurun_out/r02c_bench_n1.err
