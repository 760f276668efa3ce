#!/bin/bash
OUT=gpurun_out/s3k; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_instances.py -m gpu -q -p no:cacheprovider -k stencil > $OUT/pytest_inst.txt 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_inst.txt
V="BRO_ELL_CPV=0 BRO_ELL_CPV=1 BRO_ELL_CPV=2 BRO_ELL_CPV=0 BRO_ELL_CPV=1 BRO_ELL_CPV=2"
for c in "C5 f64" "C5 f32"; do
  timeout 900 python scripts/sweep_env.py $c ell "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
