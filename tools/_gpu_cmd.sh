export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -15 > gpurun_out/t7.log
timeout 200 python tools/quick_time.py C2 > gpurun_out/qt7_c2.log 2>&1
timeout 200 python tools/quick_time.py C3 > gpurun_out/qt7_c3.log 2>&1
for o in "--opt tile_x=32 --opt tile_y=8 --opt zchunk=64 --opt threads=64" "--opt tile_x=32 --opt tile_y=8 --opt zchunk=64 --opt threads=128" "--opt tile_x=32 --opt tile_y=16 --opt zchunk=64 --opt threads=128" "--opt tile_x=64 --opt tile_y=8 --opt zchunk=32 --opt threads=128" "--opt tile_x=32 --opt tile_y=16 --opt zchunk=32 --opt threads=64" "--opt tile_x=32 --opt tile_y=32 --opt zchunk=32 --opt threads=128" "--opt tile_x=32 --opt tile_y=8 --opt zchunk=32 --opt threads=64 --opt prefetch=2"; do
  echo "== $o" >> gpurun_out/qt7_sweep.log
  timeout 100 python tools/quick_time.py C2 fused $o 2>&1 | grep -E "fused|unfused :" >> gpurun_out/qt7_sweep.log
done
tail -3 gpurun_out/t7.log
