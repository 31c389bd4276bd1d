export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for w in C2 C3 C5; do
  timeout 900 python tools/tune_workload.py $w unfused --quick --out gpurun_out/${w}_unfused_tune.json > gpurun_out/tune_unfused_$w.log 2>&1; echo tune $w rc $?
  python tools/merge_unfused.py $w gpurun_out/${w}_unfused_tune.json && cp configs/$(echo $w | tr A-Z a-z)_plan.json gpurun_out/
done
for w in "C2 fused" "C3 measured" "C5 fused"; do set -- $w
  timeout 600 python bench.py --workload $1 --plan $2 --steps 30 --warmup 5 > gpurun_out/bench4_$1_$2.log 2>&1; tail -1 gpurun_out/bench4_$1_$2.log | cut -c1-200
done
timeout 600 python bench.py > gpurun_out/bench4_C4.log 2>&1; tail -1 gpurun_out/bench4_C4.log | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sf_ -c 200 --csv --log-file gpurun_out/launches_c4.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/b_ncu.log 2>&1; echo ncu rc $?
