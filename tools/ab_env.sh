#!/bin/bash
# Timing of the default libsg build under different environment settings on a row subset.
#   bash tools/ab_env.sh <frac> <config> "VAR=a" "VAR=b" ...
FRAC=$1; CFG=$2; shift 2
for kv in "$@"; do
  echo "== $kv"
  env $kv timeout 600 python tools/prof_rows.py --config $CFG --frac $FRAC --reps 2 2>&1 | tail -1
done
