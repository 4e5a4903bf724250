#!/bin/bash
# Time the C4 Jacobi kernels for every built libpcapps variant (PC_APPS_LIB), kernel and tile height.
cd "$(dirname "$0")/.."
for f in paper_conf_sc_temucinslsga24_b200/libpcapps.so paper_conf_sc_temucinslsga24_b200/libpcapps_m*.so; do
  [ -e "$f" ] || continue
  for kern in ${KERNELS:-rows}; do
    for h in ${HS:-64}; do
      echo -n "$(basename $f) $kern H=$h: "
      PC_APPS_LIB=$PWD/$f PC_JACOBI_KERNEL=$kern PC_JACOBI_H=$h R=1 timeout 200 python tools/jacobi_time.py 2>&1 | tail -1
    done
  done
done
