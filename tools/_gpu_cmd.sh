export PYTHONUNBUFFERED=1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q 2>&1 | tail -8 > gpurun_out/t15.log
timeout 1500 python tools/plan_autotune.py C4 --plan-from configs/c4_plan.json --tune --out gpurun_out/c4_plan_tuned.json > gpurun_out/at15.log 2>&1
cp gpurun_out/c4_plan_tuned.json configs/c4_plan.json
timeout 600 python bench.py --steps 300 --warmup 5 > gpurun_out/bench15.log 2>gpurun_out/bench15.err
tail -3 gpurun_out/t15.log; tail -12 gpurun_out/at15.log; cut -c1-300 gpurun_out/bench15.log
