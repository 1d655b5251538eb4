#!/bin/bash
# ncu --set full of one steady-state single-instance (148-SM) pipelined launch: TAG=x [ARGS=...]
T=${TAG:-single}
timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 6 -c 1 \
  -o gpurun_out/prof_single_$T -f python bench.py --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown $ARGS > gpurun_out/prof_single_$T.log 2>&1; echo rc=$?
python tools/ncu_summary.py gpurun_out/prof_single_$T.ncu-rep "" single_$T > /dev/null 2>&1; cp profiles/ncu_single_$T.md gpurun_out/ 2>/dev/null
cat gpurun_out/ncu_single_$T.md | tail -3
