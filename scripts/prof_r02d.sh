#!/bin/bash
# ncu --set full: bulk vs register-staged BRO-ELL on C5 fp64 (V = 1)
OUT=gpurun_out/r02d; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv -s 3 -c 1 \
  -o $OUT/prof_C5_f64_bulk python bench.py --workload C5 --dtype f64 --vec-words 1 --steps 6 --warmup 3 \
  --no-cpu-baseline --no-e2e > $OUT/prof_bulk.txt 2>&1; echo "bulk rc=$?"
BRO_ELL_KERNEL=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv -s 3 -c 1 \
  -o $OUT/prof_C5_f64_odv1 python bench.py --workload C5 --dtype f64 --vec-words 1 --steps 6 --warmup 3 \
  --no-cpu-baseline --no-e2e > $OUT/prof_odv1.txt 2>&1; echo "odv1 rc=$?"
