#!/bin/bash
# source-level ncu capture of the persistent kernel (sample-only call)
NCU=/usr/local/cuda/bin/ncu
timeout 1200 $NCU --set full --import-source on --clock-control none -k regex:k_csp_persistent -s 4 -c 1 \
  -o gpurun_out/src_$1 -f python tools/phases.py 6 > gpurun_out/src_$1.log 2>&1
echo rc=$?
