export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench5_C4.log 2>&1; tail -1 gpurun_out/bench5_C4.log | cut -c1-120
timeout 600 python bench.py > gpurun_out/bench5_C4b.log 2>&1; tail -1 gpurun_out/bench5_C4b.log | cut -c1-120
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench5_ref.log 2>&1; echo ref rc $?; tail -1 gpurun_out/bench5_ref.log | cut -c1-200
