#!/bin/bash
# Interleaved A/B of library variants on the biased bench step: VARIANTS="base x" REPS=2
export PYTHONUNBUFFERED=1
for rep in $(seq ${REPS:-2}); do
  for v in $VARIANTS; do
    if [ "$v" = base ]; then unset DSP_LIB; else export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so; fi
    timeout 300 python bench.py --scheme biased --steps ${STEPS:-100} --warmup 5 --no-cpu-baseline --no-breakdown $ARGS 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v rep $rep: GEPS %.3f ms/step %.4f frac %.3f' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac']))"
  done
done
