#!/bin/bash
OUT=gpurun_out/s3g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
bash scripts/ab.sh s3g "--workload C5 --dtype f32 --steps 300 --warmup 10" 2
bash scripts/ab.sh s3g "--workload C5 --steps 300 --warmup 10" 1
for ck in 1 2; do
BRO_COO_KERNEL=$ck timeout 900 ncu --set full --clock-control none --import-source on -k regex:coo_spmv -s 2 -c 1 \
  -o $OUT/prof_C4_f64_coo_k$ck python bench.py --workload C4 --format coo --steps 4 --warmup 2 --no-cpu-baseline --no-e2e > $OUT/prof_k$ck.txt 2>&1
echo "ncu k$ck rc=$?"
done
