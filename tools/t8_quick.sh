#!/bin/bash
# quick GPU check of the k_tile8 kernel: a parity subset, frame A/B at T, per-kernel times
set -x
cd "$(dirname "$0")/.."
python -c "import __graft_entry__; __graft_entry__.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "t8 and (c1 or fuzz or heavy or fig2)" 2>&1 | tail -15
timeout 300 python tools/ab_frame.py --config T --R 0 --modes t8 ws --steps 20
timeout 300 python tools/ab_frame.py --config C4 --R 15 --modes t8 ws --steps 20
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -3 | cut -c1-3000
