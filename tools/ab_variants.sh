#!/bin/bash
# A/B of experiment builds (DSP_LIB) on the default bench: VARIANTS="a b c" ROUNDS=2 bash tools/ab_variants.sh
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
for r in $(seq 1 ${ROUNDS:-2}); do
  for v in ${VARIANTS}; do
    if [ "$v" = "main" ]; then lib=""; else lib="paper_conf_ppopp_caiz0zszck23_b200/libdsp_$v.so"; fi
    DSP_LIB=$lib timeout 600 python bench.py --steps ${STEPS:-200} --warmup 5 --no-cpu-baseline $EXTRA 2> gpurun_out/ab_$v.err \
      | python -c "import json,sys; d=json.loads(sys.stdin.read()); b=d.get('breakdown') or {}; print('$v', 'round $r', round(d['ms_per_step'],5), 'frac', round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value']/1e9,3), 'gatherGBps', round(b.get('gather_GBps',0)), 'sample_ms', round(b.get('sample_call_ms_mean',0),4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
    tail -1 gpurun_out/ab_$v.err | grep -i error
  done
done
