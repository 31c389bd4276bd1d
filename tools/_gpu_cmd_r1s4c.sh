export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "c2_full or c4_full_size_bench or sampled" > gpurun_out/pytest_new.log 2>&1; echo new rc $?; tail -3 gpurun_out/pytest_new.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo all rc $?; tail -2 gpurun_out/pytest_gpu.log
