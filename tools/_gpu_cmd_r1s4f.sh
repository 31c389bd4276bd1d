export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1800 python tools/step_tune.py C4 --groups 3,5,9,1,7 --zchunks 8,16,32,64 --prefetch 1,2,3 --top 8 --out gpurun_out/c4_plan_retune.json > gpurun_out/c4_retune.log 2>&1; echo tune rc $?; grep -E "round|final|start" gpurun_out/c4_retune.log | cut -c1-200
for r in 1 2 3; do
  timeout 300 python bench.py --no-cpu --steps 200 > gpurun_out/ab_base_$r.log 2>&1; tail -1 gpurun_out/ab_base_$r.log | python -c "import json,sys; print('base', json.loads(sys.stdin.read())['ms_per_step'])"
  SF_C4_PLAN=gpurun_out/c4_plan_retune.json timeout 300 python bench.py --no-cpu --steps 200 > gpurun_out/ab_new_$r.log 2>&1; tail -1 gpurun_out/ab_new_$r.log | python -c "import json,sys; print('new', json.loads(sys.stdin.read())['ms_per_step'])"
done
