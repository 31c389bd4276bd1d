export PYTHONUNBUFFERED=1
timeout 2400 python tools/plan_autotune.py C4 --plan-from configs/c4_plan.json --tune --out gpurun_out/c4_plan_tuned3.json > gpurun_out/at19.log 2>&1
cp gpurun_out/c4_plan_tuned3.json configs/c4_plan.json
timeout 900 python bench.py --steps 500 --warmup 10 > gpurun_out/bench19.log 2>gpurun_out/bench19.err
tail -11 gpurun_out/at19.log; cut -c1-300 gpurun_out/bench19.log
