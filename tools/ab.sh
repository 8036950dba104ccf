#!/bin/bash
# A/B timing of alternative libsg builds (build_ab/libsg_*.so) on a C3 row subset; one line per build.
#   bash tools/ab.sh [frac] [config]
FRAC=${1:-0.25}; CFG=${2:-C3}
for so in paper_conf_icpp_hardhikbrks17_b200/libsg.so build_ab/libsg_*.so; do
  [ -f "$so" ] || continue
  echo "== $so"
  SG_LIB_PATH=$PWD/$so timeout 600 python tools/prof_rows.py --config $CFG --frac $FRAC --reps 2 2>&1 | tail -1
done
