OUT=gpurun_out/r02f; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
python -c "import sys; sys.path.insert(0,'scripts'); import ab_r1; ab_r1.build_r1()" > $OUT/build_r1.txt 2>&1 || echo r1 build failed
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or spmv_random or instances or single or inf" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/pytest_q.txt
timeout 900 python scripts/ab_r1.py C5 f64 "slice_h=32,ell_kernel=3" "slice_h=64,ell_kernel=10" > $OUT/ab_r1_C5_f64.txt 2>&1; grep -E "round-1|current" $OUT/ab_r1_C5_f64.txt | cut -c1-120
for dt in f64 f32; do
timeout 900 python scripts/ab.py C5 $dt "slice_h=32,ell_kernel=3" "slice_h=32,ell_kernel=6" "slice_h=32,ell_kernel=7" "slice_h=32,ell_kernel=10" "slice_h=64,ell_kernel=3" "slice_h=64,ell_kernel=6" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" "slice_h=64,ell_kernel=10" > $OUT/ab_C5_$dt.txt 2>&1; cat $OUT/ab_C5_$dt.txt
done
for T in 8 16 32; do timeout 900 python scripts/ab.py C4 f64 --format coo "coo_T=$T" --baseline-opts "coo_T=$T" > $OUT/ab_C4_coo_T$T.txt 2>&1; cat $OUT/ab_C4_coo_T$T.txt; done
for T in 8 16; do timeout 900 python scripts/ab.py C3 f64 --format coo "coo_T=$T" --baseline-opts "coo_T=$T" > $OUT/ab_C3_coo_T$T.txt 2>&1; cat $OUT/ab_C3_coo_T$T.txt; done
timeout 900 python scripts/ab.py C4 f64 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,ell_kernel=8" "slice_h=32,coo_T=8,ell_kernel=9" "slice_h=64,coo_T=8" "slice_h=64,coo_T=8,ell_kernel=9" --baseline-opts "coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt
timeout 900 python scripts/ab.py C3 f64 "slice_h=32,coo_T=8" "slice_h=64,coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C3_f64.txt 2>&1; cat $OUT/ab_C3_f64.txt
