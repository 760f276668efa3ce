OUT=gpurun_out/r02g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or instances or single or inf" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/pytest_q.txt
for dt in f64 f32; do
timeout 900 python scripts/ab.py C5 $dt "slice_h=32,ell_kernel=6" "slice_h=32,ell_kernel=7" "slice_h=32,ell_kernel=10" "slice_h=64,ell_kernel=3" "slice_h=64,ell_kernel=6" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" "slice_h=64,ell_kernel=10" > $OUT/ab_C5_$dt.txt 2>&1; cat $OUT/ab_C5_$dt.txt
done
for T in 8 16 32; do timeout 900 python scripts/ab.py C4 f64 --format coo "coo_T=$T" "coo_T=$T,coo_prefetch=2" --baseline-opts "coo_T=$T" > $OUT/ab_C4_coo_T$T.txt 2>&1; cat $OUT/ab_C4_coo_T$T.txt; done
timeout 900 python scripts/ab.py C4 f64 --format coo "coo_T=8" --baseline-opts "coo_T=8,coo_prefetch=2" > $OUT/ab_C4_coo_plainpf.txt 2>&1; cat $OUT/ab_C4_coo_plainpf.txt
for T in 8 16; do timeout 900 python scripts/ab.py C3 f64 --format coo "coo_T=$T" "coo_T=$T,coo_prefetch=2" --baseline-opts "coo_T=$T" > $OUT/ab_C3_coo_T$T.txt 2>&1; cat $OUT/ab_C3_coo_T$T.txt; done
timeout 900 python scripts/ab.py C4 f64 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,ell_kernel=8" "slice_h=32,coo_T=8,ell_kernel=9" "slice_h=64,coo_T=8" "slice_h=64,coo_T=8,ell_kernel=9" "slice_h=32,coo_T=16" --baseline-opts "coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt
timeout 900 python scripts/ab.py C4 f32 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,ell_kernel=9" "slice_h=64,coo_T=8" "slice_h=64,coo_T=8,ell_kernel=9" --baseline-opts "coo_T=8" > $OUT/ab_C4_f32.txt 2>&1; cat $OUT/ab_C4_f32.txt
