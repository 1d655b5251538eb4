#!/bin/bash
# register / spill summary of the persistent and multi kernels (ptxas -v of a fresh build)
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build(force=True, verbose=True)" 2>&1 | \
  python -c "
import sys, re
name = None
for line in sys.stdin:
    m = re.search(r\"Compiling entry function '(\S+)'\", line)
    if m: name = m.group(1); continue
    m = re.search(r'(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads', line)
    if m and name and ('persistent' in name or 'multi' in name or 'lw_' in name):
        print('%-60s stack %4s spill st %4s ld %4s' % (name[:60], *m.groups()))
"
