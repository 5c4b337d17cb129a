#!/bin/bash
# fused routing: one-process P-shard emulation tests, two processes on one GPU over CUDA IPC (gloo barriers)
OUT=gpurun_out/r3e; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_sharded.py -q -x > $OUT/sharded.log 2>&1; tail -3 $OUT/sharded.log
for r in fused nccl; do
  EIRENE_BENCH_ONE_GPU=1 timeout 900 python bench.py --gpus 2 --backend gloo --route $r --steps 5 --warmup 3 --e2e-steps 3 > $OUT/gloo2_$r.log 2>&1
  echo "== $r rc=$?"; tail -1 $OUT/gloo2_$r.log | cut -c1-400; grep -i "error\|Traceback" $OUT/gloo2_$r.log | head -5
done
