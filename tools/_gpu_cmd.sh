export PYTHONUNBUFFERED=1
timeout 900 python tools/ab_step.py C4 "pdl=0" "pdl=1" "pdl=0" "pdl=1" > gpurun_out/ab21.log 2>&1
cat gpurun_out/ab21.log
