#!/bin/bash
# L2 fetch-size qualifiers on the leaf loads: value L2::64B (v4), key line L2::128B (lp128), both
OUT=gpurun_out/r2u; mkdir -p $OUT
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
for L in libeirene.so libeirene_v4.so libeirene_lp128.so libeirene_v4lp.so; do
  EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $OUT/t_$L.csv $BENCH > /dev/null 2>&1
  echo "== $L"; python tools/traffic1.py $OUT/t_$L.csv 3 2>/dev/null | grep query
done
bash tools/ab_libs.sh r2u 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_v4.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_lp128.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_v4lp.so
