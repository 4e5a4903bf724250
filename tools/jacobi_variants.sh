#!/bin/bash
cd "$(dirname "$0")/.."
for f in paper_conf_sc_temucinslsga24_b200/libpcapps.so paper_conf_sc_temucinslsga24_b200/libpcapps_m*.so; do
  for h in 32 64; do
    echo -n "$(basename $f) H=$h: "
    PC_APPS_LIB=$PWD/$f PC_JACOBI_H=$h timeout 200 python bench.py --steps 2 --no-cpu-baseline --no-latency 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); j=d['jacobi']; print(round(j['1x1']['hbm_frac'],3), round(j['4x2']['hbm_frac'],3), round(j['1x1']['us_per_iter'],1))"
  done
done
