#!/bin/bash
OUT=gpurun_out/s4verify; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cut -c1-900 $OUT/bench.json
timeout 600 python bench.py --dtype f32 --no-cpu-baseline > $OUT/bench_C5_f32.json 2>> $OUT/bench.err; echo "f32 rc=$?"; cut -c1-600 $OUT/bench_C5_f32.json
