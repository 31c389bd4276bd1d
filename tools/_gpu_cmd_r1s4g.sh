export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "c4 or graph" > gpurun_out/pytest_c4.log 2>&1; echo c4 tests rc $?; tail -2 gpurun_out/pytest_c4.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sf_fused_5 -s 3 -c 1 -o gpurun_out/c4_fused5_r1s4g python bench.py --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu_full.log 2>&1; echo ncu rc $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sf_ -c 200 --csv --log-file gpurun_out/launches_c4g.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/b_ncu.log 2>&1; echo launches rc $?
timeout 600 python bench.py > gpurun_out/bench6_C4.log 2>&1; tail -1 gpurun_out/bench6_C4.log | cut -c1-120
