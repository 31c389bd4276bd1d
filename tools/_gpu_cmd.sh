export PYTHONUNBUFFERED=1
timeout 2400 python tools/plan_autotune.py C4 --tune --out gpurun_out/c4_plan_g.json > gpurun_out/at29.log 2>&1
SF_C4_PLAN=gpurun_out/c4_plan_g.json timeout 300 python tools/ab_step.py C4 '' '' > gpurun_out/ab29.log 2>&1
timeout 300 python tools/ab_step.py C4 '' > gpurun_out/ab29c.log 2>&1
timeout 600 python bench.py --steps 50 > gpurun_out/bench29a.log 2>&1
timeout 600 python bench.py --steps 200 > gpurun_out/bench29b.log 2>&1
cat gpurun_out/ab29.log gpurun_out/ab29c.log; grep -h -o '"ms_per_step": [0-9.]*' gpurun_out/bench29a.log gpurun_out/bench29b.log; tail -12 gpurun_out/at29.log
