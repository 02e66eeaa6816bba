#!/bin/bash
# Round profile capture (run under gpurun, 1 GPU). Writes into gpurun_out/prof_<tag>/:
#   launches.csv      ncu launch list (gpu__time_duration) of the bench command itself
#   full_<kernel>.ncu-rep   one `ncu --set full` capture per kernel family, on the bench workload
# then scripts/profile_summarize.py turns them into profiles/<tag>_*.{csv,json,txt}.
set -x
TAG=${1:-r1}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1
# full sets on the bench's fields (CESM T for SP codecs, Miranda density for DP)
for spec in "SPspeed cesm_1800x3600_f32 T speed_" "SPratio cesm_1800x3600_f32 T spratio_" \
            "DPspeed miranda_256x384x384_f64 density speed_" \
            "DPratio miranda_256x384x384_f64 density sort_|fcm_|dpratio_"; do
  set -- $spec
  ncu --set full --clock-control none --import-source on -k "regex:$4" -c 10 -o $OUT/full_$1 \
      python scripts/run_codec.py --codec $1 --config $2 --field $3 --reps 1 > $OUT/ncu_$1.log 2>&1
done
ls -la $OUT
