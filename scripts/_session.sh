set -x
bash scripts/gpu_r02.sh r02b quick
OUT=gpurun_out/r02b
timeout 900 python scripts/ab.py C5 f64 "slice_h=32,ell_kernel=3" "slice_h=32,ell_kernel=6" "slice_h=32,ell_kernel=7" "slice_h=32,ell_kernel=8" "slice_h=32,ell_kernel=9" "slice_h=64,ell_kernel=3" "slice_h=64,ell_kernel=4" "slice_h=64,ell_kernel=6" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" "slice_h=64,ell_kernel=10" > $OUT/ab_C5_f64.txt 2>&1; cat $OUT/ab_C5_f64.txt
timeout 900 python scripts/ab.py C5 f32 "slice_h=32,ell_kernel=3" "slice_h=32,ell_kernel=7" "slice_h=64,ell_kernel=3" "slice_h=64,ell_kernel=6" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" > $OUT/ab_C5_f32.txt 2>&1; cat $OUT/ab_C5_f32.txt
timeout 900 python scripts/ab.py C4 f64 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=16" > $OUT/ab_C4_coo.txt 2>&1; cat $OUT/ab_C4_coo.txt
timeout 900 python scripts/ab.py C4 f64 "slice_h=32,coo_T=16" "slice_h=64,coo_T=16" "slice_h=64,coo_T=16,ell_kernel=10" "slice_h=32,coo_T=16,ell_kernel=4" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt
timeout 900 python scripts/ab.py C3 f64 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=8" > $OUT/ab_C3_coo.txt 2>&1; cat $OUT/ab_C3_coo.txt
timeout 900 python scripts/ab.py C3 f64 "slice_h=32" "slice_h=64" > $OUT/ab_C3_f64.txt 2>&1; cat $OUT/ab_C3_f64.txt
