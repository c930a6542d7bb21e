#!/bin/bash
# parity subset + an ncu --set full capture of k_tile8 at T
cd "$(dirname "$0")/.."
python -c "import __graft_entry__; __graft_entry__.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "t8 and (c1 or fuzz or heavy or fig2)" 2>&1 | tail -5
timeout 300 python tools/ab_frame.py --config T --R 0 --modes t8 ws --steps 20
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tile8 -s 2 -c 1 -o gpurun_out/t8_full -f python tools/profile_frame.py --config T --reps 1 --tile t8 > gpurun_out/t8_ncu.log 2>&1
tail -3 gpurun_out/t8_ncu.log
