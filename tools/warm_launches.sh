#!/bin/bash
# per-kernel device times with warm caches (ncu --cache-control none): serialised
# launches, so the per-kernel numbers are comparable but not additive to the bench.
OUT=gpurun_out/warm_${1:-x}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none --csv --log-file $OUT/launches.csv \
  python tools/ab.py --reps 1 --steps 8 X=1 > $OUT/log.txt 2>&1
python tools/launches.py $OUT/launches.csv 4 | tee $OUT/summary.txt
