#!/bin/bash
# One GPU call that regenerates this round's evidence under gpurun_out/ (summarised into profiles/ afterwards):
# smoke, parity log, bench line, ncu launch list, ncu full capture of one frame, selection sweep, graph-replayed frame
# times of the paper-scale and sparse frames, and the compute-sanitizer runs.
set -u
TAG=${1:-r2}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
STARSIM_PARITY_LOG=gpurun_out/${TAG}_parity.jsonl timeout 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1
timeout 600 python bench.py > gpurun_out/${TAG}_bench_T.json 2> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python tools/profile_frame.py --reps 3 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_ -s 8 -c 4 -f -o gpurun_out/${TAG}_full \
  python tools/profile_frame.py --reps 1 > gpurun_out/ncu_full.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tile_wide -s 2 -c 1 -f \
  -o gpurun_out/${TAG}_wide_R63 python tools/profile_frame.py --config C4 --R 63 --reps 1 > gpurun_out/ncu_wide.log 2>&1
timeout 900 python tools/sweep.py --sweep all > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/sweep.err
for c in "C1 0" "fig2 0" "C2 0" "C3 1000" "C3 16000" "C3 100000" "C4 0" "T 0"; do
  set -- $c; timeout 120 python tools/frame_time.py --config $1 --n $2
done > gpurun_out/${TAG}_frames.txt 2>&1
S=/usr/local/cuda/bin/compute-sanitizer
for t in memcheck synccheck initcheck; do
  timeout 900 $S --tool $t --print-limit 20 python tools/sanitize_run.py > gpurun_out/${TAG}_sanitize_$t.log 2>&1
done
timeout 900 $S --tool racecheck --racecheck-report all --print-limit 20 python tools/sanitize_run.py --quick \
  > gpurun_out/${TAG}_sanitize_racecheck_all.log 2>&1
for k in lists sb ws t8; do
  timeout 600 $S --tool racecheck --racecheck-report all --print-limit 20 python tools/sanitize_run.py --quick \
    --kernels=$k > gpurun_out/${TAG}_sanitize_racecheck_$k.log 2>&1
done
tail -2 gpurun_out/gpu_tests.log
