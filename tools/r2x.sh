#!/bin/bash
# steady-state L2 behaviour of the query kernel by eviction policy (single pass, no cache flush)
OUT=gpurun_out/r2x; mkdir -p $OUT
BENCH="python bench.py --steps 8 --warmup 3 --e2e-steps 0 --cpu-batches 0 --ra-probe 0"
M=gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_evict_last_lookup_hit.sum,lts__t_sectors_srcunit_tex_evict_last_lookup_miss.sum,lts__t_sectors_srcunit_tex_evict_first_lookup_hit.sum,lts__t_sectors_srcunit_tex_evict_first_lookup_miss.sum,lts__t_sectors_srcunit_tex_evict_normal_lookup_hit.sum,lts__t_sectors_srcunit_tex_evict_normal_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum
timeout 600 ncu --metrics $M -k regex:query_kernel --cache-control none --clock-control none --csv --log-file $OUT/pol.csv $BENCH > /dev/null 2>&1
python - <<'PY'
import csv,collections
rows=list(csv.reader(open('gpurun_out/r2x/pol.csv')))
hi=next(i for i,r in enumerate(rows) if 'Kernel Name' in r); h=rows[hi]
ii,mi,vi=h.index('ID'),h.index('Metric Name'),h.index('Metric Value')
per=collections.defaultdict(dict)
for r in rows[hi+1:]:
    if len(r)>vi: per[r[ii]][r[mi]]=float(r[vi].replace(',',''))
ids=sorted(per,key=int)[3:]
for m in sorted(per[ids[0]]):
    v=sorted(per[i][m] for i in ids); print(f"{m:70s} median {v[len(v)//2]:.4g}")
PY
