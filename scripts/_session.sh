set -x
bash scripts/gpu_r02.sh r02a quick
OUT=gpurun_out/r02a
timeout 600 python scripts/ab.py C5 f64 "slice_h=32" "slice_h=64" "slice_h=64,ell_kernel=4" "slice_h=64,ell_kernel=5" > $OUT/ab_C5_f64.txt 2>&1; cat $OUT/ab_C5_f64.txt | tail -6
timeout 600 python scripts/ab.py C5 f32 "slice_h=32" "slice_h=64" "slice_h=64,ell_kernel=4" > $OUT/ab_C5_f32.txt 2>&1; cat $OUT/ab_C5_f32.txt | tail -5
timeout 600 python scripts/ab.py C4 f64 "slice_h=32,coo_T=32" "slice_h=64,coo_T=32" "slice_h=64,coo_T=16" "slice_h=64,coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt | tail -6
timeout 600 python scripts/ab.py C4 f32 "slice_h=32" "slice_h=64" > $OUT/ab_C4_f32.txt 2>&1; cat $OUT/ab_C4_f32.txt | tail -4
timeout 600 python scripts/ab.py C4 f64 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=32" > $OUT/ab_C4_coo.txt 2>&1; cat $OUT/ab_C4_coo.txt | tail -5
timeout 600 python scripts/ab.py C3 f64 "slice_h=32" "slice_h=64" "slice_h=64,coo_T=16" > $OUT/ab_C3_f64.txt 2>&1; cat $OUT/ab_C3_f64.txt | tail -5
timeout 600 python scripts/ab.py C3 f64 --format coo "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=8" > $OUT/ab_C3_coo.txt 2>&1; cat $OUT/ab_C3_coo.txt | tail -5
timeout 600 python scripts/ab.py C2 f64 "slice_h=32" "slice_h=64" "slice_h=32,ell_kernel=5" > $OUT/ab_C2_f64.txt 2>&1; cat $OUT/ab_C2_f64.txt | tail -5
