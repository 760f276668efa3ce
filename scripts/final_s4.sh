#!/bin/bash
# Session-4 final evidence (after the .L2::256B streamed-load hint): GPU tests, smoke,
# default bench, all configs, ncu launch list + full capture of the default kernel
OUT=gpurun_out/final_s4; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
for wl in C1 C2 C3 C4 C5; do for dt in f64 f32; do
  fl=""; [ $wl = C1 -o $wl = C2 -o $wl = C3 ] && fl="--flush-l2"
  timeout 600 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/bench_all.err
  echo "$wl $dt rc=$?"; done; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
  --log-file $OUT/launches_C5.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.txt 2>&1
echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv_od -s 3 -c 1 \
  -o $OUT/prof_C5_f64 python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full.txt 2>&1
echo "ncu full rc=$?"
