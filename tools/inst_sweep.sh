#!/bin/bash
export PYTHONUNBUFFERED=1
q() { timeout 900 python bench.py --steps ${STEPS:-200} --warmup 5 --no-cpu-baseline --no-breakdown "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ms/step %.4f frac %.3f' % (d['ms_per_step'], d['roofline']['frac']))"; }
for r in 1 2; do
  echo -n "products inst2 lw5: "; q --instances 2
  echo -n "products inst2 lw4: "; DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_lw4.so q --instances 2
done
for sc in layer; do for i in 2 4; do echo -n "$sc inst$i: "; q --scheme $sc --instances $i; done; done
for cfg in papers friendster; do for i in 2 4; do echo -n "$cfg inst$i: "; STEPS=50 q --config $cfg --instances $i; done; done
