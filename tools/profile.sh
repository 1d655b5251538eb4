#!/bin/bash
# ncu evidence for the default bench configuration (1 GPU).  $1 = tag, $2 = kernel regex
tag=${1:-r01}
kre=${2:-"k_"}
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
# 1) every launch with its device time (cold-cache, serialised): compare shares, not absolutes
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_${tag}.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline $BENCH_ARGS \
  > gpurun_out/launches_${tag}.log 2>&1
echo "launch list rc=$?"
# 2) full sections for steady-state launches of the top kernels
timeout 1500 $NCU --set full --clock-control none --import-source on \
  -k regex:"${kre}" -s ${SKIP:-6} -c ${COUNT:-3} -o gpurun_out/prof_${tag} -f \
  python bench.py --steps 12 --warmup 3 --no-cpu-baseline $BENCH_ARGS > gpurun_out/prof_${tag}.log 2>&1
echo "full rc=$?"
# 3) the bench line itself (no profiler)
python bench.py $BENCH_ARGS > gpurun_out/bench_${tag}.json 2> gpurun_out/bench_${tag}.err
echo "bench rc=$?"; tail -c 600 gpurun_out/bench_${tag}.json
