#!/bin/bash
# Round checkpoint on one B200: GPU parity suite, smoke, default bench line, reference arm,
# per-config sweep (+ iteration-warp ablation, cfg5 at N=1), ncu launch list + full capture
# of the hot kernels, warm-cache traffic of the query kernel.
TAG=${1:-x}
OUT=gpurun_out/ckpt_$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.log 2>&1
CFGS="1 3 4 6" BENCH_ARGS="--e2e-steps 0 --cpu-batches 1 --ra-probe 0" bash tools/allcfg.sh $TAG > $OUT/allcfg.txt 2>&1
timeout 600 python bench.py --query-mode iterwarp --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/bench_iterwarp.log 2>&1
timeout 1200 python bench.py --config 5 --steps 10 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/bench_cfg5.log 2>&1
timeout 900 bash tools_profile.sh $TAG > $OUT/profile.log 2>&1
timeout 600 bash tools/ncu_traffic.sh $TAG > $OUT/traffic.log 2>&1
tail -3 $OUT/gpu_tests.log; tail -1 $OUT/smoke.log; cat $OUT/allcfg.txt
tail -1 $OUT/bench.log | cut -c1-300
