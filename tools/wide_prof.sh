#!/bin/bash
# k_tile_wide: parity tests, C4 ROI-sweep timings (auto vs lists), one ncu --set full capture per R.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "wide or c4 or circle_roi or fuzz or heavy" > gpurun_out/wide_tests.log 2>&1
tail -3 gpurun_out/wide_tests.log
for R in 21 31 47 63; do
  for m in auto lists; do timeout 120 python tools/ab_kern.py --config C4 --R $R --mode $m; done
done > gpurun_out/wide_ab.txt 2>&1
cat gpurun_out/wide_ab.txt
for R in ${PROF_R:-63 31}; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tile_wide -s 2 -c 1 -f \
    -o gpurun_out/wide_R$R python tools/profile_frame.py --config C4 --R $R --reps 1 > gpurun_out/ncu_wide_R$R.log 2>&1
done
