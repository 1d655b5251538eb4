export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_red_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_red.sum
for inst in 1 4; do
timeout 900 /usr/local/cuda/bin/ncu --cache-control none --clock-control none --metrics $M -k regex:k_csp -s 10 -c 3 --csv --log-file gpurun_out/warm2_i$inst.csv python bench.py --steps 16 --warmup 3 --no-cpu-baseline --no-breakdown --instances $inst > /dev/null 2>&1; echo rc=$?
done
