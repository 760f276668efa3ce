#!/bin/bash
OUT=gpurun_out/s3n; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="- BRO_ELL_VARIANT=2 BRO_ELL_VARIANT=3 BRO_ELL_VARIANT=4 BRO_ELL_VARIANT=5 -"
for c in "C5 f32" "C5 f64"; do
  timeout 900 python scripts/sweep_env.py $c ell "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
