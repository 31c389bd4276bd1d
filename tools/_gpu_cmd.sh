export PYTHONUNBUFFERED=1
timeout 300 python tools/ab_step.py C4 'factor=0' 'factor=1' 'factor=0' 'factor=1' > gpurun_out/ab27.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "c4 or parity_vs" 2>&1 | tail -3 > gpurun_out/t27.log
timeout 2400 python tools/plan_autotune.py C4 --tune --out gpurun_out/c4_plan_f.json > gpurun_out/at27.log 2>&1
SF_C4_PLAN=gpurun_out/c4_plan_f.json timeout 300 python tools/ab_step.py C4 '' '' > gpurun_out/ab27b.log 2>&1
cat gpurun_out/ab27.log gpurun_out/t27.log gpurun_out/ab27b.log; tail -20 gpurun_out/at27.log
