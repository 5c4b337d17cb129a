#!/bin/bash
# result-store variants of the query kernel (EIRENE_RES_ST 0 / 1 / 2): single-pass DRAM traffic and A/B
OUT=gpurun_out/r2p; mkdir -p $OUT
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
for L in libeirene.so libeirene_rs1.so libeirene_rs2.so; do
  EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $OUT/t_$L.csv $BENCH > /dev/null 2>&1
  echo "== $L"; python tools/traffic1.py $OUT/t_$L.csv 3 | head -6
done
bash tools/ab_libs.sh r2p 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_rs1.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_rs2.so
