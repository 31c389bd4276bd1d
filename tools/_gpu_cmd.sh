export PYTHONUNBUFFERED=1
for w in "C2 fused" "C3 measured" "C3 fission_fused" "C3 fused" "C5 fused"; do set -- $w
  timeout 600 python bench.py --workload $1 --plan $2 --steps 30 --warmup 5 > gpurun_out/bench3_$1_$2.log 2>&1; tail -1 gpurun_out/bench3_$1_$2.log | cut -c1-150
done
timeout 600 python bench.py > gpurun_out/bench3_C4.log 2>&1; tail -1 gpurun_out/bench3_C4.log | cut -c1-150
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sf_ -c 200 --csv --log-file gpurun_out/launches_c4.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/b_ncu.log 2>&1
