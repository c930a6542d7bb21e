#!/bin/bash
# 1,024-star binning blocks for small catalogues (current build) vs 4,096 everywhere (libstarsim_binold.so)
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "bins or heavy or routed or c4 or fuzz or unsplit or c1 or fig2 or full_frame or sparse or band" > gpurun_out/binsmall_tests.log 2>&1
tail -1 gpurun_out/binsmall_tests.log
for i in 1 2; do
for c in "C3 8192 0" "C3 16384 0" "C3 65536 0" "C3 262144 0" "C2 0 0" "C4 0 15" "C4 0 63" "T 0 0"; do
  set -- $c
  timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3
  STARSIM_LIB=$P/libstarsim_binold.so timeout 120 python tools/frame_time.py --config $1 --n $2 --R $3 | sed 's/^/old /'
done
done
