#!/bin/bash
# update kernel ALU: binary-search ranks; batched runs with the plan kept -- parity, A/B cfg4 / cfg1 (head / nobatch / batch)
OUT=gpurun_out/r3g; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_key32.py -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab_libs.sh r3g4 4 $P/libeirene_head.so $P/libeirene_nobatch.so $P/libeirene.so
bash tools/ab_libs.sh r3g1 1 $P/libeirene_head.so $P/libeirene_nobatch.so $P/libeirene.so
