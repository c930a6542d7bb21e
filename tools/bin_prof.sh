#!/bin/bash
# ncu --set full of the binning kernels and the tile kernel at T (one frame), for source-level hotspots
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_dcount|k_dplace|k_dcolscan|k_tile_ws" -s 8 -c 4 -f \
  -o gpurun_out/binT python tools/profile_frame.py --reps 1 > gpurun_out/ncu_binT.log 2>&1
tail -3 gpurun_out/ncu_binT.log
