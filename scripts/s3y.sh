#!/bin/bash
OUT=gpurun_out/s3y; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.txt
for wl in C1 C2 C3 C4; do for dt in f64 f32; do
  fl=""; [ $wl = C1 -o $wl = C2 -o $wl = C3 ] && fl="--flush-l2"
  timeout 600 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/bench_all.err
  echo "$wl $dt rc=$?"; done; done
timeout 600 python bench.py --workload C5 --steps 500 --no-cpu-baseline > $OUT/bench_C5_f64.json 2>> $OUT/bench_all.err; echo "C5 rc=$?"
