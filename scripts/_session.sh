OUT=gpurun_out/r02c; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or spmv_random" > $OUT/pytest_coo.txt 2>&1; echo "coo tests rc=$?"; tail -3 $OUT/pytest_coo.txt
timeout 900 python scripts/ab_r1.py C5 f64 "slice_h=32,ell_kernel=3" "slice_h=32,ell_kernel=7" > $OUT/ab_r1_C5_f64.txt 2>&1; cat $OUT/ab_r1_C5_f64.txt | grep -v "^nvcc\|ptxas" | cut -c1-250
timeout 900 python scripts/ab.py C4 f64 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=16" > $OUT/ab_C4_coo.txt 2>&1; cat $OUT/ab_C4_coo.txt
timeout 900 python scripts/ab.py C4 f32 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=16" > $OUT/ab_C4_coo32.txt 2>&1; cat $OUT/ab_C4_coo32.txt
timeout 900 python scripts/ab.py C3 f64 --format coo "coo_T=8" "coo_T=16" --baseline-opts "coo_T=8" > $OUT/ab_C3_coo.txt 2>&1; cat $OUT/ab_C3_coo.txt
timeout 900 python scripts/ab.py C4 f64 "slice_h=32,coo_T=16" "slice_h=32,coo_T=16,ell_kernel=10" "slice_h=32,coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt
