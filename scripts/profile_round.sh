#!/bin/bash
# Round profile capture (run under gpurun, 1 GPU). Writes into gpurun_out/prof_<tag>/:
#   launches.csv      ncu launch list (gpu__time_duration) of the bench command itself
#   full_<codec>_<field>.ncu-rep   `ncu --set full` captures per kernel family on the
#                     bench's largest fields (NYX 512³ velocity for the SP codecs:
#                     2 GiB of traffic, far beyond the 126 MB L2; Miranda rt_density
#                     and density for the DP codecs)
# then scripts/profile_summarize.py turns them into profiles/<tag>_*.{csv,json,txt}.
set -x
TAG=${1:-r2}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-transfer > $OUT/bench_under_ncu.log 2>&1
for spec in "SPspeed nyx_512x512x512_f32 velocity speed_" "SPratio nyx_512x512x512_f32 velocity spratio_" \
            "DPspeed miranda_256x384x384_f64 density speed_" \
            "DPratio miranda_256x384x384_f64 rt_density sort_|fcm_|dpratio_|dp_" \
            "DPratio miranda_256x384x384_f64 density dpratio_"; do
  set -- $spec
  ncu --set full --clock-control none --import-source on -k "regex:$4" -c 12 -o $OUT/full_$1_$3 \
      python scripts/run_codec.py --codec $1 --config $2 --field $3 --reps 1 > $OUT/ncu_$1_$3.log 2>&1
done
ls -la $OUT
