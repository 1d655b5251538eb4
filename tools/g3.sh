export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
for bps in 8 2 1; do echo "bps $bps"; DSP_STAGE_BPS=$bps P=2 timeout 300 python tools/virtual_time.py 2>&1 | tail -1; done
echo "gpu-scope fence"; DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_gf.so P=2 timeout 300 python tools/virtual_time.py 2>&1 | tail -1
P=8 timeout 300 python tools/virtual_time.py 2>&1 | tail -3
bash tools/profile.sh r01g k_csp
