#!/bin/bash
# Interleaved A/B of library variants on the bench headline: VARIANTS="base x" REPS=3 [ARGS="--instances 4"]
export PYTHONUNBUFFERED=1
for rep in $(seq ${REPS:-3}); do
  for v in $VARIANTS; do
    if [ "$v" = base ]; then unset DSP_LIB; else export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so; fi
    timeout 300 python bench.py --steps ${STEPS:-300} --warmup 5 --no-cpu-baseline --no-breakdown $ARGS 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v rep $rep: GEPS %.3f ms/step %.4f frac %.3f clk %s' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz']))"
  done
done
