bash scripts/run_sweep.sh r01e "0" "C5:f64:0,1,3,8 C5:f32:0,1,3,8 C2:f64:0,1,8 C4:f64:0,1 C4:f32:0,1 C2:f32:0,1" "spmv_random or vec_words or decode or config5_full or single_long or inf or config4"
bash scripts/prof.sh r01e C5 f64 0 bro_ell_spmv_od
bash scripts/prof.sh r01e C5 f64 0 "^ell_spmv"
