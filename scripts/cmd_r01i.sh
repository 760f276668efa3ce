bash scripts/run_sweep.sh r01i "0" "C4:f64:0 C4:f32:0 C3:f64:0 C3:f32:0 C5:f64:0" "spmv_random or decode or single_long or inf or config4 or configs_full or determin or side_stream"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01i/launches_C3.csv python bench.py --workload C3 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --flush-l2 > /dev/null 2>&1; echo "launches C3 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01i/launches_C4.csv python bench.py --workload C4 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "launches C4 rc=$?"
bash scripts/prof.sh r01i C4 f64 0 coo_spmv
