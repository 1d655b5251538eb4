#!/bin/bash
# ncu captures of steady-state launches (a pipelined launch that gathers the previous batch),
# the standalone gather, and the walk / layer-wise kernels.  1 GPU, never multi-rank.
export PYTHONUNBUFFERED=1
T=${TAG:-r02}
NCU=/usr/local/cuda/bin/ncu
M=--set\ full
# bench config (4 streams x 37 SMs): skip 3 warm-up launches + 3 flush gathers + the 4 first timed launches
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 7 -c 2 \
  -o gpurun_out/prof_$T -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_$T.log 2>&1; echo "bench4 rc=$?"
# single instance on all 148 SMs
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 6 -c 1 \
  -o gpurun_out/prof_single_$T -f python bench.py --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_single_$T.log 2>&1; echo "single rc=$?"
# the standalone gather
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_gather_tma" -s 4 -c 1 \
  -o gpurun_out/prof_gather_$T -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline > gpurun_out/prof_gather_$T.log 2>&1; echo "gather rc=$?"
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_random_walk" -s 4 -c 1 \
  -o gpurun_out/prof_walk_$T -f python bench.py --scheme walk --steps 8 --warmup 3 --no-cpu-baseline > gpurun_out/prof_walk_$T.log 2>&1; echo "walk rc=$?"
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_lw_persistent" -s 8 -c 1 \
  -o gpurun_out/prof_layer_$T -f python bench.py --scheme layer --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_layer_$T.log 2>&1; echo "layer rc=$?"
# summaries here (the reports are large); keep only the single-instance capture
for t in $T single_$T gather_$T walk_$T layer_$T; do
  python tools/ncu_summary.py gpurun_out/prof_$t.ncu-rep "" $t > /dev/null 2>&1 && cp profiles/ncu_$t.md gpurun_out/ 2>/dev/null
done
cp profiles/ncu_traffic.json gpurun_out/ncu_traffic_box.json
rm -f gpurun_out/prof_$T.ncu-rep gpurun_out/prof_gather_$T.ncu-rep gpurun_out/prof_walk_$T.ncu-rep gpurun_out/prof_layer_$T.ncu-rep
ls -la gpurun_out/
