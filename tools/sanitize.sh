#!/bin/bash
# compute-sanitizer over the tiny-config GPU paths (persistent kernel, pipelined, virtual ranks)
CS=/usr/local/cuda/bin/compute-sanitizer
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 1200 $CS --tool $tool --error-exitcode 9 --print-limit 20 python -m pytest -x -q \
    tests/test_gpu_parity.py -k "fanout_range or sample_gather_sync or pipelined_steps or tiny_virtual_ranks or fig5 or errors" \
    2>&1 | tail -6
  echo "rc=${PIPESTATUS[0]}"
done
