#!/bin/bash
# One GPU call that regenerates this round's evidence under gpurun_out/ (copied to profiles/ by hand):
# bench line, parity log, ncu launch list, ncu full capture of one frame, C3/C4 selection sweep.
set -u
TAG=${1:-r1b}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
STARSIM_PARITY_LOG=gpurun_out/${TAG}_parity.jsonl timeout 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1
timeout 400 python bench.py > gpurun_out/${TAG}_bench_T.json 2> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python tools/profile_frame.py --reps 3 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_ -s 8 -c 4 -f -o gpurun_out/${TAG}_full \
  python tools/profile_frame.py --reps 1 > gpurun_out/ncu_full.log 2>&1
timeout 900 python tools/sweep.py --sweep all > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/sweep.err
tail -2 gpurun_out/gpu_tests.log
