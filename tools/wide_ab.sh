#!/bin/bash
# k_tile_wide / binning: parity tests, then per-kernel-class device times on the C4 ROI sweep and T.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-wide or c4 or circle_roi or fuzz or heavy or bins or routed}" > gpurun_out/wide_tests.log 2>&1
tail -3 gpurun_out/wide_tests.log
for R in ${RS:-3 9 15 21 31 47 63}; do
  for m in ${MODES:-auto lists}; do timeout 120 python tools/ab_kern.py --config C4 --R $R --mode $m; done
done > gpurun_out/wide_ab.txt 2>&1
timeout 120 python tools/ab_kern.py --config T --mode auto >> gpurun_out/wide_ab.txt 2>&1
cat gpurun_out/wide_ab.txt
