#!/bin/bash
# Engine tuning sweep (N=1, 8 virtual ranks): one bench line per knob setting.
cd "$(dirname "$0")/.."
run() {
  echo "== $*"
  env "$@" timeout 120 python bench.py --steps 50 --warmup 5 --no-latency --no-jacobi --no-cpu-baseline --e2e-steps 1 $EXTRA 2>/dev/null \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; c=d['config']; print(f\"busbw {d['value']:.1f} GB/s  ms {d['ms_per_step']:.3f}  engine_ms {r['engine_ms']:.3f} frac {r['frac']:.3f}  slices {c['slices_per_chunk']} slice_elems {c['slice_elems']} warps {c['engine_warps_per_rank']}\")"
}
for kv in "$@"; do
  run $kv
done
