#!/bin/bash
# same-box A/B of k_tile_sb variants (libstarsim_<NAME>.so) in mode sb at T, C4 R=15, C3 262K
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for c in "T 0" "C4 0" "C3 262144"; do
  set -- $c
  timeout 120 python tools/ab_kern.py --config $1 --n $2 --mode sb
  timeout 120 python tools/ab_kern.py --config $1 --n $2 --mode ws
  for v in $VARS; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config $1 --n $2 --mode sb; done
done
done
