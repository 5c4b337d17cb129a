#!/bin/bash
# contention probe of the leaf allocation counter (EIRENE_ALLOC_DIAG: striped counters, holes)
OUT=gpurun_out/r3a; mkdir -p $OUT
P=paper_conf_ppopp_zhangz0lzl23_b200
for L in libeirene.so libeirene_adiag.so; do
  EIRENE_LIB=$P/$L EIRENE_UPDATE_PROF=1 timeout 600 python bench.py --config 4 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0 > $OUT/$L.log 2>&1
  echo "== $L"; grep "upd prof" $OUT/$L.log | tail -3; tail -1 $OUT/$L.log | cut -c1-150
done
