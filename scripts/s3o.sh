#!/bin/bash
# A/B/C: libbro.so (tail + meta pointers) vs libbro_ab.so (tail only) vs libbro_ab2.so (before)
OUT=gpurun_out/s3o; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
for r in 1 2; do for lib in libbro.so libbro_ab.so libbro_ab2.so; do
  BRO_LIB=$lib timeout 900 python scripts/sweep_env.py C5 f64 ell "-" 300 2>&1 | sed "s/^/$lib /" | tee -a $OUT/sweep.txt | grep -v Warn
  BRO_LIB=$lib timeout 900 python scripts/sweep_env.py C5 f32 ell "-" 300 2>&1 | sed "s/^/$lib /" | tee -a $OUT/sweep.txt | grep -v Warn
done; done
