#!/bin/bash
# DRAM bytes per launch without cache flushes: sampling only, fused sample+gather, the bench configuration
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build()" || exit 1
for m in sample sample_gather pipelined; do echo "== $m"; MODES=$m bash tools/ncu_steady.sh $m; done
NCU=/usr/local/cuda/bin/ncu
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum
echo "== bench config"
timeout 900 $NCU --metrics $M --cache-control none --clock-control none -k regex:k_csp_persistent -s 20 -c 4 --csv python bench.py --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/steady_bench.csv 2>gpurun_out/steady_bench.err
grep -v "^==" gpurun_out/steady_bench.csv | grep -v '^{' | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin))
h=rows[0]
for r in rows[1:]:
    d=dict(zip(h,r)); print(d.get('ID'), d.get('Metric Name'), d.get('Metric Unit'), d.get('Metric Value'))
"
