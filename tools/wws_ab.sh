#!/bin/bash
# same-box A/B: k_tile_wide (sb) vs k_tile_wws (ws) and variants on C4 wide ROIs
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for R in 31 47 63; do
  for m in sb ws; do timeout 120 python tools/ab_kern.py --config C4 --R $R --mode $m; done
  for v in "$@"; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/ab_kern.py --config C4 --R $R --mode ws; done
done
