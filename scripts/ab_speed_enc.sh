#!/bin/bash
# A/B of speed-codec library variants (args: .so paths), median of 9.
cd "$(dirname "$0")/.."
for L in "$@"; do
  for c in "SPspeed nyx_512x512x512_f32 velocity" "DPspeed miranda_256x384x384_f64 density" "SPspeed cesm_1800x3600_f32 T"; do
    set -- $c
    LCF_LIB_PATH=$L python scripts/ab_time.py --codec $1 --config $2 --field $3 --reps 9
  done
done
