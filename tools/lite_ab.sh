#!/bin/bash
# k_tile_lite with per-star slots (current build) vs the per-lane profile evaluation (libstarsim_liteold.so)
P=paper_conf_ipps_lizzh12_b200
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "ws_equals_sb or sparse or circle or integrated or c1 or fig2 or fuzz" > gpurun_out/lite_tests.log 2>&1
tail -2 gpurun_out/lite_tests.log
for i in 1 2; do
for c in "C3 4096" "C3 8192" "C3 16384" "C3 32768" "C2 0"; do
  set -- $c
  timeout 120 python tools/frame_time.py --config $1 --n $2
  STARSIM_LIB=$P/libstarsim_liteold.so timeout 120 python tools/frame_time.py --config $1 --n $2 | sed 's/^/old /'
done
done
