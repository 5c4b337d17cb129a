#!/bin/bash
# iteration-warp ablation: GPU tests + bench lines; cfg5 at N=1
OUT=gpurun_out/iw_${1:-x}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_iterwarp.py -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
tail -3 $OUT/tests.log
for it in 0 4 16; do
  timeout 300 python bench.py --query-mode iterwarp --iter-rgs $it --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 > $OUT/bench_iw$it.log 2>&1
  tail -1 $OUT/bench_iw$it.log | cut -c1-200; tail -1 $OUT/bench_iw$it.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['stage_ms'], d['traversal'], d['parity'])"
done
timeout 1200 python bench.py --config 5 --steps 10 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/bench_cfg5.log 2>&1; echo "rc=$?"
tail -3 $OUT/bench_cfg5.log | cut -c1-1500
