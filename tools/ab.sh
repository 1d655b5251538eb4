#!/bin/bash
# A/B of library variants on one box, interleaved: VARIANTS="base ih" (base = libdsp.so)
export PYTHONUNBUFFERED=1
for rep in 1 2; do
  for v in $VARIANTS; do
    if [ "$v" = base ]; then unset DSP_LIB; else export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so; fi
    echo "== $v (rep $rep)"
    DIM=4 KS=4 timeout 300 python tools/instances.py 2>&1 | grep "pipelined=False"
    KS=3 timeout 300 python tools/instances.py 2>&1 | grep "pipelined=True"
  done
done
