#!/bin/bash
# count-matrix block threshold variants (libstarsim_<NAME>.so) on mid-size and full frames
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for c in "C3 393216 0" "C3 524288 0" "C3 786432 0" "T 0 0" "C5 0 0"; do
  set -- $c
  timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3 --steps 10
  for v in $VARS; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3 --steps 10 | sed "s/^/$v /"; done
done
done
