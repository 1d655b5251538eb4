#!/bin/bash
# biased phases of library variants: VARIANTS="base x y"
export PYTHONUNBUFFERED=1
for v in ${VARIANTS:-base}; do
  if [ "$v" = base ]; then unset DSP_LIB; else export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so; fi
  echo "== $v"; MODES=${MODES:-biased} timeout 300 python tools/phases.py 12 2>&1 | grep -v "^  pipelined" | head -12
done
