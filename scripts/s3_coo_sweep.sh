#!/bin/bash
OUT=gpurun_out/s3d; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="- BRO_COO_UPI=1 BRO_COO_UPI=4 BRO_COO_MINB=4 BRO_COO_MINB=4,BRO_COO_UPI=4 BRO_COO_MINB=4,BRO_COO_UPI=1"
for c in "C3 f64" "C3 f32" "C4 f64" "C4 f32"; do
  timeout 900 python scripts/sweep_env.py $c hyb,coo "$V" 200 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
