#!/bin/bash
# launch lists (C3, C4 f64) + ncu --set full of C4's BRO-ELL and BRO-COO kernels
OUT=gpurun_out/r02g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
for wl in C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv \
    --log-file $OUT/launches_${wl}.csv python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
  echo "launches $wl rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv -s 3 -c 1 \
  -o $OUT/prof_C4_f64_ell python bench.py --workload C4 --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "ell rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:coo_spmv -s 3 -c 1 \
  -o $OUT/prof_C4_f64_coo python bench.py --workload C4 --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "coo rc=$?"
