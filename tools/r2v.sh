#!/bin/bash
# value loads with a 64 B L2 fetch (default now); key-line loads L2::64B (lp64): GPU suite, traffic, A/B
OUT=gpurun_out/r2v; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
for L in libeirene_head.so libeirene.so libeirene_lp64.so; do
  EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $OUT/t_$L.csv $BENCH > /dev/null 2>&1
  echo "== $L"; python tools/traffic1.py $OUT/t_$L.csv 3 2>/dev/null | grep -E "query|group|dist"
done
bash tools/ab_libs.sh r2v 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene_lp64.so
bash tools/ab_libs.sh r2v3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
