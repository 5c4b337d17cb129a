#!/bin/bash
# chunk claims G at a time + per-warp level-0 count (update), QCOOP default: full GPU suite, A/B vs HEAD
OUT=gpurun_out/r3i; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab2.sh r3i4 4 10 2 $P/libeirene_head.so $P/libeirene.so
bash tools/ab2.sh r3i1 1 20 2 $P/libeirene_head.so $P/libeirene.so
bash tools/ab2.sh r3i2 2 20 2 $P/libeirene_head.so $P/libeirene.so
timeout 300 python bench.py --config 7 --steps 20 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg7.log 2>&1; tail -1 $OUT/cfg7.log | cut -c1-200
