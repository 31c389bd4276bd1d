export PYTHONUNBUFFERED=1
timeout 700 python tools/sweep.py C4 --group 2 --grid --tx 32,64,128,256 --zchunk 32 --pf 1,2,3 > gpurun_out/sw2_g2.log 2>&1
timeout 700 python tools/sweep.py C4 --group 5 --grid --tx 32,64,128 --zchunk 32 --pf 2,3 > gpurun_out/sw2_g5.log 2>&1
tail -3 gpurun_out/sw2_g2.log
