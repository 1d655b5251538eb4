#!/bin/bash
# Records the GPU box's host and device properties into gpurun_out/box_probe.txt
out=gpurun_out/box_probe.txt
{
  echo "== nproc"; nproc
  echo "== affinity"; python -c 'import os; print(len(os.sched_getaffinity(0)))'
  echo "== lscpu"; lscpu | head -20
  echo "== free -g"; free -g
  echo "== nvidia-smi"; nvidia-smi
  echo "== topo"; nvidia-smi topo -m
  echo "== torch"; python -c '
import torch
p = torch.cuda.get_device_properties(0)
print(p)
print("l2", p.L2_cache_size, "sms", p.multi_processor_count)
'
  echo "== df /tmp"; df -h /tmp
} > $out 2>&1
cat $out | head -80
