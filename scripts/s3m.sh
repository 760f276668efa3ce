#!/bin/bash
OUT=gpurun_out/s3m; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="BRO_COO_L2PF=1 BRO_COO_L2PF=0 BRO_COO_L2PF=1 BRO_COO_L2PF=0"
for c in "C4 f64" "C4 f32" "C3 f64"; do
  timeout 900 python scripts/sweep_env.py $c hyb,coo "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
  BRO_LIB=libbro_ab.so timeout 900 python scripts/sweep_env.py $c hyb,coo "- -" 300 2>&1 | sed 's/^/AB(prev) /' | tee -a $OUT/sweep.txt | grep -v Warn
done
