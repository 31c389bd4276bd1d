export PYTHONUNBUFFERED=1
timeout 300 python tools/step_series.py C4 --steps 600 --window 20 > gpurun_out/ser31.log 2>&1
timeout 300 python tools/step_series.py C4 --steps 400 --window 20 --mode unfused > gpurun_out/ser31u.log 2>&1
nvidia-smi -q -d POWER,CLOCK,PERFORMANCE > gpurun_out/smi31.txt 2>&1
head -2 gpurun_out/ser31.log; head -2 gpurun_out/ser31u.log
