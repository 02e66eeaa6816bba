#!/bin/bash
# A/B timing matrix: every library given on the command line × the bench's
# codec/config pairs (scripts/ab_time.py, median of 7).
cd "$(dirname "$0")/.."
for L in "$@"; do
  for c in "SPspeed nyx_512x512x512_f32 velocity" "SPratio nyx_512x512x512_f32 velocity" \
           "DPspeed miranda_256x384x384_f64 density" "DPratio miranda_256x384x384_f64 density" \
           "SPspeed cesm_1800x3600_f32 T" "SPratio cesm_1800x3600_f32 T"; do
    set -- $c
    LCF_LIB_PATH=$L python scripts/ab_time.py --codec $1 --config $2 --field $3 --reps 7
  done
done
