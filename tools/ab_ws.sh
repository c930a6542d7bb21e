#!/bin/bash
# warp-specialised tile kernel diagnostics: ms/frame and tile ms for the default build, the sb kernel, and the
# consumer-less / profile-less builds (tile kernel only)
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
run() { timeout 300 python bench.py --steps 30 --no-e2e --no-cpu-baseline "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step']*1000,2), round(d['kernels']['tile']['ms_per_step']*1000,2))"; }
for i in 1 2; do
  echo "ws   $(run)"
  echo "sb   $(run --tile-kernel sb)"
  for v in $@; do echo "$v $(STARSIM_LIB=$P/libstarsim_$v.so run)"; done
done
