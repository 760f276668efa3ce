#!/bin/bash
# session-3 check: GPU parity after the COO decode changes + C3/C4 benches
TAG=${1:-s3a}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.txt
for wl in C3 C4; do for dt in f64 f32; do
  fl=""; [ $wl = C3 ] && fl="--flush-l2"
  timeout 600 python bench.py --workload $wl --dtype $dt --steps 300 --no-cpu-baseline --no-e2e $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/bench.err
  echo "$wl $dt rc=$?"; python -c "import json,sys; d=json.load(open('$OUT/bench_${wl}_${dt}.json')); print(d['value'], d['roofline']['frac'], d.get('uncompressed',{}))"
  timeout 600 python bench.py --workload $wl --dtype $dt --format coo --steps 300 --no-cpu-baseline --no-e2e $fl > $OUT/bench_${wl}_${dt}_coo.json 2>> $OUT/bench.err
  echo "$wl $dt coo rc=$?"; python -c "import json,sys; d=json.load(open('$OUT/bench_${wl}_${dt}_coo.json')); print(d['value'], d['roofline']['frac'], d.get('uncompressed',{}))"
done; done
