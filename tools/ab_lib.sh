#!/bin/bash
# same-box A/B of the current build against paper_conf_ipps_lizzh12_b200/libstarsim_<NAME>.so for each NAME given:
# ms/frame and the tile kernel's ms at T, two rounds
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
run() { timeout 300 python bench.py --steps 30 --no-e2e --no-cpu-baseline "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step']*1000,2), round(d['kernels']['tile']['ms_per_step']*1000,2))"; }
for i in 1 2; do
  echo "cur $(run)"
  for v in $@; do echo "$v $(STARSIM_LIB=$P/libstarsim_$v.so run)"; done
done
