export PYTHONUNBUFFERED=1
timeout 900 python tools/sweep.py C2 --group 0 --grid --tx 32,64 --zchunk 8,16,32,64 --pf 2 > gpurun_out/sw_c2.log 2>&1
timeout 900 python tools/sweep.py C3 --plan-name fission_fused --group 0 --grid --tx 64,128 --zchunk 8,16,32 --pf 2 > gpurun_out/sw_c3.log 2>&1
timeout 900 python tools/sweep.py C5 --group 0 --grid --tx 32,64 --zchunk 8,16,32 --pf 2 > gpurun_out/sw_c5.log 2>&1
