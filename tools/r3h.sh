#!/bin/bash
# query kernel: warp-cooperative leaf search A/B (cfg2, cfg7-like off); update kernel ncu capture under cfg4
OUT=gpurun_out/r3h; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
bash tools/ab2.sh r3h2 2 20 2 $P/libeirene.so $P/libeirene_qcoop.so
EIRENE_LIB=$P/libeirene_qcoop.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "query or fig3 or cfg2 or tiny or host" > $OUT/qcoop_tests.log 2>&1; tail -2 $OUT/qcoop_tests.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel -s 4 -c 1 -o $OUT/upd4 \
  python bench.py --config 4 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/upd4.log 2>&1
python tools/ncu_lines.py $OUT/upd4.ncu-rep update_kernel 40 > $OUT/ncu_lines_upd4.txt 2>&1; head -45 $OUT/ncu_lines_upd4.txt
python tools/ncu_summary.py $OUT/upd4.ncu-rep > $OUT/ncu_upd4_summary.txt 2>&1; cat $OUT/ncu_upd4_summary.txt
