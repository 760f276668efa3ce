#!/bin/bash
OUT=gpurun_out/s3i; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="BRO_ELL_FEW_G=0 BRO_ELL_FEW_G=16 BRO_ELL_FEW_G=32"
for c in "C2 f64" "C2 f32" "C1 f64" "C1 f32"; do
  timeout 900 python scripts/sweep_env.py $c ell "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?"; tail -5 $OUT/pytest_gpu.txt
