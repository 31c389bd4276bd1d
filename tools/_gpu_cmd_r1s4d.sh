export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sf_fused_5 -s 3 -c 1 -o gpurun_out/c4_fused5_r1s4 python bench.py --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu_full.log 2>&1; echo ncu rc $?
timeout 1500 python tools/step_tune.py C2 --zchunks 4,8,16,32,64 --prefetch 1,2,3 --top 10 > gpurun_out/c2_step_tune.log 2>&1; echo tune rc $?; tail -3 gpurun_out/c2_step_tune.log
