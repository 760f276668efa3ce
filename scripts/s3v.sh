#!/bin/bash
OUT=gpurun_out/s3v; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python scripts/sweep_env.py C5 f64 ell "- BRO_ELL_VARIANT=6 BRO_ELL_VARIANT=7 - BRO_ELL_VARIANT=6 BRO_ELL_VARIANT=7" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
timeout 900 python scripts/sweep_env.py C5 f32 ell "- BRO_ELL_VARIANT=6 BRO_ELL_VARIANT=7" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
timeout 900 python scripts/sweep_env.py C4 f64 hyb "- BRO_ELL_SMALLWIN=0 -" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
