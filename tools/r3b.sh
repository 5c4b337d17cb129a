#!/bin/bash
# query kernel: child-line L1 prefetch A/B (EIRENE_CHILD_PF); phase profile of the distribution and group kernels (cfg2)
OUT=gpurun_out/r3b; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
EIRENE_LIB=$P/libeirene_phase.so timeout 300 python tools/phase_prof.py 2 > $OUT/phase2.txt 2>&1; cat $OUT/phase2.txt
bash tools/ab_libs.sh r3b2 2 $P/libeirene.so $P/libeirene_cpf.so
