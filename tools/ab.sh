#!/bin/bash
# A/B timing of two library builds on the same box: tools/ab.sh <libA.so> <libB.so> [rounds]
# (built in-tree beforehand; prints ms/frame and the tile kernel's ms for each round)
A=$1; B=$2; N=${3:-3}
for i in $(seq 1 $N); do
  for L in $A $B; do
    STARSIM_LIB=$L timeout 300 python bench.py --steps 30 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$L', round(d['ms_per_step']*1000,2), round(d['kernels']['tile']['ms_per_step']*1000,2))"
  done
done
