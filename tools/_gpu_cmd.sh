export PYTHONUNBUFFERED=1
mkdir -p gpurun_out/dump
for o in "loader=1" "loader=0"; do
  timeout 120 python tools/debug_one.py chain3 unfused $o fmad=0 >> gpurun_out/dbg.log 2>&1
  timeout 120 python tools/debug_one.py chain3 fused $o fmad=0 >> gpurun_out/dbg.log 2>&1
  timeout 120 python tools/debug_one.py C2 fused $o fmad=0 >> gpurun_out/dbg.log 2>&1
  timeout 120 python tools/debug_one.py C3 fission_fused $o fmad=0 >> gpurun_out/dbg.log 2>&1
done
SF_DUMP_DIR=gpurun_out/dump CUDA_LAUNCH_BLOCKING=1 timeout 300 compute-sanitizer --tool memcheck --show-backtrace device python tools/debug_one.py chain3 unfused loader=0 > gpurun_out/san.log 2>&1
tail -5 gpurun_out/dbg.log
