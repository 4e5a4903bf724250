#!/bin/bash
# last measurement set of the round: GPU suite (default and system scope), smoke, bench, C2 / latency legs
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -3 > gpurun_out/r02g_pytest_gpu.txt
PC_FORCE_SYS_SCOPE=1 timeout 1200 python -m pytest tests -x -q -m gpu -p no:cacheprovider 2>&1 | tail -3 > gpurun_out/r02g_sys_scope_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02g_smoke.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02g_bench_n1.json 2> gpurun_out/r02g_bench_n1.err
PC_FORCE_SYS_SCOPE=1 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02g_bench_sys_scope.json 2>/dev/null
timeout 600 python tools/sweep.py p2p --batched --graph --persistent --sizes 1048576,16777216,67108864,268435456 --grans block_put --aggs none > gpurun_out/r02g_c2.jsonl 2>/dev/null
cat gpurun_out/r02g_pytest_gpu.txt gpurun_out/r02g_sys_scope_pytest.txt; tail -1 gpurun_out/r02g_smoke.txt
for f in gpurun_out/r02g_bench_n1.json gpurun_out/r02g_bench_sys_scope.json; do python - "$f" <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read())
print(sys.argv[1], round(d["value"],1), d["clocks"], {k: (v.get("p50") if isinstance(v, dict) else v) for k, v in d["latency_ns"].items() if k != "note"},
      "c1", round(d["c1_p2p"]["partitioned_us_device"],1), "c2", round(d["c2_p2p_256mib"]["partitioned_us"],1), round(d["c2_p2p_256mib"]["traditional_us"],1))
PY
done
python - <<'PY'
import json
for l in open("gpurun_out/r02g_c2.jsonl"):
    d=json.loads(l)
    if d.get("copy")=="engine": continue
    print(d["bytes"]>>20, d.get("mode","put")[:11], round(d["us"],1), d.get("parity",""))
PY
