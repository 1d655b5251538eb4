#!/bin/bash
# steady-state (no cache flush between kernels) DRAM/L2 counters of the persistent kernel
# usage: MODES=sample bash tools/ncu_steady.sh tag
NCU=/usr/local/cuda/bin/ncu
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_atom_dot_alu_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_atom_dot_alu_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_write_lookup_miss.sum
timeout 600 $NCU --metrics $M --cache-control none --clock-control none -k regex:k_csp_persistent -s 6 -c 3 --csv \
  python tools/phases.py 10 > gpurun_out/steady_$1.csv 2> gpurun_out/steady_$1.err
echo rc=$?
grep -v "^==" gpurun_out/steady_$1.csv | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin))
h=rows[0]
for r in rows[1:]:
    d=dict(zip(h,r)); print(d.get('ID'), d.get('Metric Name'), d.get('Metric Unit'), d.get('Metric Value'))
"
