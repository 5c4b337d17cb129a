#!/bin/bash
# Copy a checkpoint's summaries (gpurun_out/ckpt_TAG, from tools/checkpoint.sh) into profiles/ as PREFIX_*.
TAG=$1; P=${2:-r2}; O=gpurun_out/ckpt_$TAG
set -e
cp $O/gpu_tests.log profiles/${P}_gpu_tests.log
cp $O/smoke.log profiles/${P}_smoke.log
grep -q "ERROR SUMMARY: 0" $O/sanitize.txt 2>/dev/null && cp $O/sanitize.txt profiles/${P}_sanitize.txt || true   # compute-sanitizer closed on the pool since r2b
cp $O/launches.csv profiles/${P}_launches.csv
cp $O/launches_summary.txt profiles/${P}_launches_summary.txt
cp $O/traffic1.txt profiles/${P}_traffic1.txt
cp $O/ncu_full_summary.txt profiles/${P}_ncu_full_summary.txt
cp $O/ncu_source_query.txt profiles/${P}_ncu_source_query.txt
for k in query group dist; do [ -f $O/ncu_lines_$k.txt ] && cp $O/ncu_lines_$k.txt profiles/${P}_ncu_lines_$k.txt; done
cp $O/pcie_bw.txt profiles/${P}_pcie_bw.txt
cp $O/gpu.txt profiles/${P}_gpu.txt
[ -f $O/traffic.json ] && cp $O/traffic.json profiles/traffic.json
tail -1 $O/bench.log > profiles/${P}_bench.json
tail -1 $O/bench_ref.log > profiles/${P}_bench_reference.json
tail -1 $O/gloo2.log > profiles/${P}_gloo2.json
: > profiles/${P}_allcfg.txt
for f in cfg1 cfg3 cfg4 cfg6 cfg7 cfg2_pipeline cfg2_iterwarp cfg5A cfg5B cfg5C cfg5U; do echo "$f $(tail -1 $O/$f.log)" >> profiles/${P}_allcfg.txt; done
