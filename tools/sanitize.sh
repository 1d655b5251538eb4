#!/bin/bash
# compute-sanitizer over the tiny-config GPU paths: world-1 persistent kernel (plain,
# fused, pipelined), every relabel-map layout incl. window crossings.  The sanitizer
# serialises kernels, so the world > 1 persistent kernels (whose ranks wait on each
# other inside the kernel) cannot run under it: virtual-rank tests are deselected.
CS=/usr/local/cuda/bin/compute-sanitizer
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 2400 $CS --tool $tool --error-exitcode 9 --print-limit 20 python -m pytest -x -q \
    tests/test_gpu_parity.py tests/test_gpu_relabel_hash.py tests/test_gpu_layerwise.py tests/test_gpu_tiered.py \
    -k "(fanout_range or sample_gather_sync or pipelined_steps or tiny_virtual_ranks or fig5 or errors or tag_wrap or fused_and_pipelined or duplicate_seed or layerwise_tiny_p1 or big_tasks or concurrent_streams or long_rows or random_walks_tiny or split_rows_layout or tiered_gather_p1 or (random_walks_independent and 1)) and not virtual" \
    2>&1 | tail -6
  echo "rc=${PIPESTATUS[0]}"
done
