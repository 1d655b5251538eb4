#!/bin/bash
# A/B of library variants on the synchronous fused call (tools/sync_overhead.py): VARIANTS="head base"
export PYTHONUNBUFFERED=1
for rep in $(seq ${REPS:-2}); do
  for v in $VARIANTS; do
    if [ "$v" = base ]; then unset DSP_LIB; else export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so; fi
    echo -n "$v rep $rep: "; timeout 300 python tools/sync_overhead.py 2>&1 | tail -1
  done
done
