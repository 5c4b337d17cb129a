#!/bin/bash
OUT=gpurun_out/grpp_${1:-x}
mkdir -p $OUT
EIRENE_GROUP_PROF=1 timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg3_prof.log 2>&1
grep "mode 2" $OUT/cfg3_prof.log | head -20
python tools/grp_parse.py $OUT/cfg3_prof.log
ncu --set full --clock-control none --import-source on -k regex:group_kernel -s 3 -c 1 -o $OUT/grp3 python bench.py --config 3 --steps 1 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/ncu.log 2>&1
