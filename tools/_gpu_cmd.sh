export PYTHONUNBUFFERED=1
timeout 1200 python tools/ab_step.py C4 "l2pf=0" "l2pf=2" "l2pf=4" "l2pf=8" "l2pf=0" > gpurun_out/ab25.log 2>&1
for g in 5 3; do timeout 300 python tools/sweep.py C4 --group $g --apply-tuning --cfg l2pf=0 --cfg l2pf=2 --cfg l2pf=4 --cfg l2pf=8 >> gpurun_out/sw25.log 2>&1; done
cat gpurun_out/ab25.log; grep -E "l2pf" gpurun_out/sw25.log | cut -c1-130
