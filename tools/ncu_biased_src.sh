#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${TAG:-s4}
echo "== ncu biased src"; MODES=biased timeout 900 /usr/local/cuda/bin/ncu --set full --import-source on --clock-control none -k regex:k_csp_persistent -s 4 -c 1 -o gpurun_out/src_biased_$T -f python tools/phases.py 6 > gpurun_out/src_biased_$T.log 2>&1; echo rc=$?
