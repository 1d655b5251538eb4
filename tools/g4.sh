export PYTHONUNBUFFERED=1
for P in 2 8; do for v in base gf base gf; do if [ $v = gf ]; then export DSP_LIB=$PWD/paper_conf_ppopp_caiz0zszck23_b200/libdsp_gf.so; else unset DSP_LIB; fi; echo "$v"; P=$P timeout 300 python tools/virtual_time.py 2>&1 | tail -1; P=$P timeout 300 python tools/phases_multi.py 2>&1 | tail -2; done; done
