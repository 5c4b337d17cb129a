#!/bin/bash
OUT=gpurun_out/fuse_${1:-x}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
tail -3 $OUT/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
for c in 2 3; do
  timeout 300 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg$c.log 2>&1
  tail -1 $OUT/cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity']['mismatches'], d['gpu_launches'])"
done
EIRENE_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --backend gloo --steps 5 --warmup 3 > $OUT/gloo2.log 2>&1; echo "gloo2 rc=$?"
tail -1 $OUT/gloo2.log | cut -c1-400
