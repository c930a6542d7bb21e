#!/bin/bash
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "heavy or unsplit or c4 or wide" > gpurun_out/red_tests.log 2>&1; tail -1 gpurun_out/red_tests.log
for i in 1 2; do
for R in 15 31 47 63; do
  timeout 120 python tools/ab_kern.py --config C4 --R $R --mode auto
  for v in $VARS; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config C4 --R $R --mode auto; done
done
done
