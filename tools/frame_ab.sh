#!/bin/bash
# graph-replayed frame times of prebuilt variants: tools/frame_ab.sh "base nolite" "C3:1000 C3:16000 C1:0 C2:0 fig2:0 T:0"
cd "$(dirname "$0")/.."
for c in $2; do
  IFS=: read -r cfg n R <<< "$c"
  for v in $1; do
    STARSIM_LIB=paper_conf_ipps_lizzh12_b200/libstarsim_$v.so timeout 300 python tools/frame_time.py --config "$cfg" \
      --n "${n:-0}" --R "${R:-0}" | sed "s/^/$v /"
  done
done
