#!/bin/bash
OUT=gpurun_out/s3h; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="- BRO_ELL_VARIANT=2 BRO_ELL_VARIANT=3 BRO_ELL_VARIANT=4 BRO_ELL_VARIANT=1"
for c in "C2 f64" "C2 f32" "C1 f64" "C4 f64" "C4 f32"; do
  f=ell; [ "${c:0:2}" = C4 ] && f=hyb
  timeout 900 python scripts/sweep_env.py $c $f "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
