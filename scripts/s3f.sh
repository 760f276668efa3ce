#!/bin/bash
OUT=gpurun_out/s3f; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_coo_pipe.py -m gpu -q -x -p no:cacheprovider > $OUT/pytest_pipe.txt 2>&1
echo "pytest pipe rc=$?"; tail -15 $OUT/pytest_pipe.txt
V="BRO_COO_KERNEL=1 BRO_COO_KERNEL=1,BRO_COO_MINB=4 BRO_COO_KERNEL=2 BRO_COO_KERNEL=2,BRO_COO_PIPE_MINB=3"
for c in "C4 f64" "C4 f32" "C3 f64" "C3 f32"; do
  timeout 900 python scripts/sweep_env.py $c hyb,coo "$V" 200 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
