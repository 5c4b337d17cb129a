#!/bin/bash
# Round checkpoint on one B200 (everything committed under profiles/ comes from here):
# GPU parity suite + smoke, the default bench line, the reference arm, a per-config sweep
# (cfg1/3/4/6/7, pipelined cfg2, iteration-warp ablation, cfg5 mixes at N=1), the N=2
# code path on one GPU (gloo, key-slice parity), compute-sanitizer, the ncu launch list,
# single-pass steady-state traffic (-> profiles/traffic.json), full captures of the hot
# kernels, PCIe copy bandwidth.
TAG=${1:-x}
OUT=gpurun_out/ckpt_$TAG
mkdir -p $OUT
SHA=${SHA:-unknown}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
python -m paper_conf_ppopp_zhangz0lzl23_b200.build > $OUT/build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q > $OUT/gpu_tests.log 2>&1; echo "rc=$?" >> $OUT/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
# single-pass steady-state traffic first: the bench line reads profiles/traffic.json of this commit
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
  --clock-control none --csv --log-file $OUT/traffic.csv $BENCH > $OUT/traffic.log 2>&1
python tools/traffic1.py $OUT/traffic.csv 3 > $OUT/traffic1.txt 2>&1
python tools/traffic_json.py $OUT/traffic.csv $TAG $SHA > $OUT/traffic_json.log 2>&1; cp profiles/traffic.json $OUT/ 2>/dev/null
timeout 900 python bench.py > $OUT/bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.log 2>&1
A="--e2e-steps 0 --cpu-batches 1 --ra-probe 0 --steps 20 --warmup 5"
for c in 1 3 4 6 7; do timeout 600 python bench.py --config $c $A > $OUT/cfg$c.log 2>&1; done
timeout 600 python bench.py --pipeline 1 $A > $OUT/cfg2_pipeline.log 2>&1
timeout 600 python bench.py --query-mode iterwarp $A > $OUT/cfg2_iterwarp.log 2>&1
for m in A B C U; do timeout 1500 python bench.py --config 5 --mix $m --steps 5 --warmup 3 --e2e-steps 0 --cpu-batches 1 --ra-probe 0 > $OUT/cfg5$m.log 2>&1; done
EIRENE_BENCH_ONE_GPU=1 timeout 900 python bench.py --gpus 2 --backend gloo --steps 5 --warmup 3 --e2e-steps 3 > $OUT/gloo2.log 2>&1
# compute-sanitizer is closed on this pool since r2b (profiles/r2_sanitize.txt is the r2a run)
[ -n "$SANITIZE" ] && timeout 1500 bash tools/sanitize.sh $TAG > $OUT/sanitize.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/launches.log 2>&1
python tools/launches.py $OUT/launches.csv 3 > $OUT/launches_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:query_kernel|group_kernel|bsort_dist|update_kernel" \
  -s 12 -c 4 -o $OUT/full $BENCH > $OUT/full.log 2>&1
python tools/ncu_summary.py $OUT/full.ncu-rep > $OUT/ncu_full_summary.txt 2>&1
python tools/ncu_source.py $OUT/full.ncu-rep query_kernel 30 > $OUT/ncu_source_query.txt 2>&1
python tools/ncu_lines.py $OUT/full.ncu-rep query_kernel 30 > $OUT/ncu_lines_query.txt 2>&1
python tools/ncu_lines.py $OUT/full.ncu-rep group_kernel 30 > $OUT/ncu_lines_group.txt 2>&1
python tools/ncu_lines.py $OUT/full.ncu-rep bsort_dist_kernel 30 > $OUT/ncu_lines_dist.txt 2>&1
timeout 120 python tools/pcie_bw.py > $OUT/pcie_bw.txt 2>&1
tail -3 $OUT/gpu_tests.log; tail -2 $OUT/smoke.log; cat $OUT/launches_summary.txt | head -8
cat $OUT/traffic_json.log
for f in bench cfg1 cfg3 cfg4 cfg6 cfg7 cfg2_pipeline cfg2_iterwarp cfg5A cfg5B cfg5C cfg5U gloo2 bench_ref; do tail -1 $OUT/$f.log | python -c "
import json,sys
try:
    d=json.loads(sys.stdin.read())
    st=d.get('stage_ms') or {}
    print('$f', round(d['value'],4), d['unit'], 'ms/step', round(d['ms_per_step']*1e3,1), {k: round(v*1e3,1) for k,v in st.items()}, 'var', d.get('batch_ms') and round(d['batch_ms']['variance_maxmin_over_mean'],3), 'parity', (d.get('parity') or {}).get('mismatches'), 'e2e', d.get('e2e') and d['e2e'].get('value'))
except Exception as e: print('$f FAILED', e)"; done
cat $OUT/pcie_bw.txt
