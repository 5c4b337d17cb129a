#!/bin/bash
# query kernel DRAM traffic composition: no value load (qd1), no leaf loads (qd2), no result stores (RES_ST=2)
OUT=gpurun_out/r2t; mkdir -p $OUT
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
for L in libeirene.so libeirene_qd1.so libeirene_qd2.so; do
  EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum --cache-control none --clock-control none --csv --log-file $OUT/t_$L.csv $BENCH > /dev/null 2>&1
  echo "== $L"; python tools/traffic1.py $OUT/t_$L.csv 3 2>/dev/null | grep query
done
