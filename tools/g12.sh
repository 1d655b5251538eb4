export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_red_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_red.sum
for pm in 0 64 1000; do
DSP_L2_PERSIST_MB=$pm timeout 900 /usr/local/cuda/bin/ncu --cache-control none --clock-control none --metrics $M -k regex:k_csp -s 10 -c 2 --csv --log-file gpurun_out/warm_pm$pm.csv python bench.py --steps 16 --warmup 3 --no-cpu-baseline --no-breakdown --instances 1 > /dev/null 2> gpurun_out/warm_pm$pm.err; echo rc=$?; grep "persisting" gpurun_out/warm_pm$pm.err | head -1
done
for rep in 1 2; do for pm in 0 32 64 1000; do DSP_L2_PERSIST_MB=$pm ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed "s/^/pm $pm /"; done; done
