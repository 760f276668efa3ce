#!/bin/bash
# source-level ncu captures: C5 f32/f64 BRO-ELL kernel, C4 f64 BRO-COO part
TAG=${1:-s3p}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
for dt in f32 f64; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv_od -s 3 -c 1 \
    -o $OUT/prof_C5_${dt} python bench.py --workload C5 --dtype $dt --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/prof_C5_${dt}.txt 2>&1
  echo "C5 $dt rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:coo_spmv -s 3 -c 1 \
  -o $OUT/prof_C4_f64_coo python bench.py --workload C4 --dtype f64 --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/prof_C4_coo.txt 2>&1
echo "C4 coo rc=$?"
