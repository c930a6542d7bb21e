#!/bin/bash
# same-box A/B of wide-ROI variants (libstarsim_<NAME>.so) on the C4 ROI sweep and a uniform wide-ROI field
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for R in 19 21 25 31 47 63; do
  timeout 120 python tools/ab_kern.py --config C4 --R $R --mode lists
  timeout 120 python tools/ab_kern.py --config C4 --R $R --mode auto
  for v in "$@"; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config C4 --R $R --mode auto; done
done
for R in 21 31 63; do
  timeout 120 python tools/ab_kern.py --config T --R $R --n 200000 --mode lists
  timeout 120 python tools/ab_kern.py --config T --R $R --n 200000 --mode auto
  for v in "$@"; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config T --R $R --n 200000 --mode auto; done
done
