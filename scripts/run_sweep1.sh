#!/bin/bash
OUT=gpurun_out/r01b
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { cat $OUT/build.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "spmv_random or vec_words or decode or config5_full or single_long or inf" > $OUT/pytest.txt 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest.txt
python scripts/sweep.py $OUT "0 1 2 3 4 5" "C5:f64 C5:f32" 2>&1
python scripts/sweep.py $OUT "0 1 3" "C2:f64 C4:f64" 2>&1
