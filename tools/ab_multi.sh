#!/bin/bash
# same-box A/B of prebuilt library variants (paper_conf_ipps_lizzh12_b200/libstarsim_NAME.so, built on the CPU side
# with STARSIM_NVCC_EXTRA) over several frames: tools/ab_multi.sh "name1 name2" "T:sb C3:auto:0:1000 C4:lists:63"
cd "$(dirname "$0")/.."
for c in $2; do
  IFS=: read -r cfg mode R n <<< "$c"
  for v in $1; do
    STARSIM_LIB=paper_conf_ipps_lizzh12_b200/libstarsim_$v.so timeout 300 python tools/ab_kern.py --config "$cfg" \
      --mode "${mode:-auto}" --R "${R:-0}" --n "${n:-0}" | sed "s/^/$v /"
  done
done
