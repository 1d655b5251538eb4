export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_relabel_hash.py -x -q -k "virtual or fig5" 2>&1 | tail -2
for P in 2 4 8; do P=$P timeout 300 python tools/virtual_time.py 2>&1 | tail -1; P=$P timeout 300 python tools/phases_multi.py 2>&1 | tail -2; done
timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -2
