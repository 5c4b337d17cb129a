#!/bin/bash
# update kernel early exit (nothing left: CTA 0 publishes): GPU suite, A/B cfg2 / cfg3; group / dist phase profile
OUT=gpurun_out/r2r; mkdir -p $OUT
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -2 $OUT/gpu_tests.log
bash tools/ab_libs.sh r2r 2 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
bash tools/ab_libs.sh r2r3 3 paper_conf_ppopp_zhangz0lzl23_b200/libeirene_head.so paper_conf_ppopp_zhangz0lzl23_b200/libeirene.so
EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_phase.so timeout 300 python tools/phase_prof.py 2 > $OUT/phase_cfg2.txt 2>&1; cat $OUT/phase_cfg2.txt
