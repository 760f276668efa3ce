bash scripts/run_sweep.sh r01d "0" "C5:f64:0,1,2,3,4,8 C5:f32:0,2,3,8 C2:f64:0,4,8 C4:f64:0,8 C4:f32:0,8" "spmv_random or vec_words or decode or config5_full or single_long or inf or config4 or configs_full_oracle and 2"
bash scripts/prof.sh r01d C5 f64 0 bro_ell_spmv_tma
bash scripts/prof.sh r01d C5 f64 8 bro_ell_spmv
