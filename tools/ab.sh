#!/bin/bash
# A/B of two library builds on the same box: tools/ab.sh CONFIG libA libB [reps]
cfg=$1; A=$2; B=$3; n=${4:-2}
for i in $(seq $n); do
  for L in $A $B; do
    echo -n "$(basename $L) "; OOO_LIB=$L timeout 300 python tools/engine_sweep.py $cfg "" 2>&1 | grep variant
  done
done
