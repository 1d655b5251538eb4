#!/bin/bash
# ncu evidence for one bench configuration (1 GPU).  $1 = tag (e.g. r01), $2 = kernel regex
tag=${1:-r01}
kre=${2:-"k_"}
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
# 1) every launch with its device time (cold-cache, serialised): compare shares
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_${tag}.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
  > gpurun_out/launches_${tag}.log 2>&1
echo "launch list rc=$?"
# 2) full sections for the kernels of one steady-state step
timeout 1500 $NCU --set full --clock-control none --import-source on \
  -k regex:"${kre}" -s ${SKIP:-4} -c ${COUNT:-3} -o gpurun_out/prof_${tag} -f \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/prof_${tag}.log 2>&1
echo "full rc=$?"
ls -la gpurun_out
