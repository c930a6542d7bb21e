#!/bin/bash
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for c in "C4 31 0" "C4 47 0" "T 31 200000" "T 47 200000"; do
  set -- $c
  timeout 120 python tools/ab_kern.py --config $1 --R $2 --n $3 --mode auto
  for v in $VARS; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config $1 --R $2 --n $3 --mode auto; done
done
done
