#!/bin/bash
# A/B timing of alternative libsg builds (build_ab/libsg_*.so, e.g. -DSG_D2_EXP timing experiments)
# against the default build with tools/ab_variant.py; one line per build.
#   bash tools/ab_builds.sh [frac] [config] [settings]
FRAC=${1:-0.25}; CFG=${2:-C3}; SET=${3:-0:-1}
for so in paper_conf_icpp_hardhikbrks17_b200/libsg.so build_ab/libsg_*.so; do
  [ -f "$so" ] || continue
  echo "== $so"
  SG_LIB_PATH=$PWD/$so timeout 600 python tools/ab_variant.py --config $CFG --frac $FRAC --settings $SET --reps 2 2>&1 | tail -1
done
