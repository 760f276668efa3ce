OUT=gpurun_out/r02p; mkdir -p $OUT
bash scripts/gpu_r02.sh r02p tests smoke bench benchall launches
for wl in C3 C4; do for dt in f64 f32; do
  fl=""; [ $wl = C3 ] && fl="--flush-l2"
  timeout 600 python bench.py --workload $wl --dtype $dt --format coo --steps 500 --no-cpu-baseline --no-e2e $fl > $OUT/bench_${wl}_${dt}_coo.json 2>> $OUT/benchcoo.err; echo "$wl $dt coo rc=$?"
done; done
for wl in C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file $OUT/launches_$wl.csv python scripts/prof_one.py $wl f64 --launches 10 > /dev/null 2>&1; python scripts/launch_summary.py $OUT/launches_$wl.csv
done
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 50 --warmup 5 --workload C2 --dist-backend gloo --no-e2e > $OUT/bench_gloo2_C2.json 2> $OUT/bench_gloo2.err; echo "gloo2 rc=$?"; cut -c1-600 $OUT/bench_gloo2_C2.json
