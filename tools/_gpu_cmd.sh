export PYTHONUNBUFFERED=1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sf_ --csv --log-file gpurun_out/launches9.csv python tools/prof_step.py C4 --steps 2 --warmup 1 --unfused > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sf_fused_0 -c 1 -o gpurun_out/prof_c4f0 python tools/prof_step.py C4 --steps 1 --warmup 0 > gpurun_out/ncu9.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sf_fused_6 -c 1 -o gpurun_out/prof_c4f6 python tools/prof_step.py C4 --steps 1 --warmup 0 >> gpurun_out/ncu9.log 2>&1
tail -2 gpurun_out/ncu9.log
