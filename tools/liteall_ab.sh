#!/bin/bash
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for c in "C4 0 3" "C4 0 9" "C4 0 15" "C3 65536 0" "C3 131072 0" "C3 262144 0" "T 0 0"; do
  set -- $c
  timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3 --steps 10
  for v in $VARS; do STARSIM_LIB=$P/libstarsim_$v.so timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3 --steps 10 | sed "s/^/$v /"; done
done
done
