#!/bin/bash
OUT=gpurun_out/bins_${1:-x}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/tests.log 2>&1; echo "rc=$?" >> $OUT/tests.log
tail -3 $OUT/tests.log
for c in 2 3; do
  timeout 300 python bench.py --config $c --steps 30 --warmup 5 --e2e-steps 0 --cpu-batches 1 > $OUT/cfg$c.log 2>&1
  tail -1 $OUT/cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg', d['config']['cfg'], round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()}, d['parity'])"
done
timeout 600 python bench.py --config 5 --tree 16777216 --steps 5 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg5s.log 2>&1
tail -1 $OUT/cfg5s.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg5s', round(d['value'],3), {k: round(v*1e3,1) for k,v in d['stage_ms'].items()})"
EIRENE_GROUP_PROF=1 timeout 600 python bench.py --config 5 --tree 16777216 --steps 3 --warmup 3 --e2e-steps 0 --cpu-batches 0 > $OUT/cfg5s_prof.log 2>&1
grep -c "group prof" $OUT/cfg5s_prof.log; grep "group prof" $OUT/cfg5s_prof.log | sort -k11 -g -r | head -4; grep "group prof" $OUT/cfg5s_prof.log | sort -k15 -g -r | head -4
