OUT=gpurun_out/r02k; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "instances or forced" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -2 $OUT/pytest_q.txt
timeout 900 python scripts/ab.py C5 f64 "slice_h=32" "slice_h=32,ell_kernel=6" "slice_h=64" "slice_h=64,ell_kernel=6" > $OUT/ab_C5_f64.txt 2>&1; cat $OUT/ab_C5_f64.txt
timeout 900 python scripts/ab.py C5 f32 "slice_h=32" "slice_h=32,ell_kernel=6" "slice_h=64" "slice_h=64,ell_kernel=6" > $OUT/ab_C5_f32.txt 2>&1; cat $OUT/ab_C5_f32.txt
for dt in f64 f32; do
timeout 900 python scripts/ab.py C4 $dt "slice_h=32" "slice_h=32,ell_kernel=7" "slice_h=32,ell_kernel=8" "slice_h=32,ell_kernel=9" "slice_h=32,ell_kernel=10" "slice_h=64" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" "slice_h=64,ell_kernel=9" "slice_h=64,ell_kernel=10" > $OUT/ab_C4_$dt.txt 2>&1; cat $OUT/ab_C4_$dt.txt
done
