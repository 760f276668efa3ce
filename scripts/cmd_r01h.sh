bash scripts/run_sweep.sh r01h "0" "C5:f64:0 C5:f32:0 C4:f64:0 C4:f32:0 C3:f64:0 C3:f32:0 C2:f64:0 C2:f32:0 C1:f64:0" "spmv_random or vec_words or decode or config5_full or single_long or inf or config4 or configs_full or determin"
bash scripts/prof.sh r01h C5 f32 0 bro_ell_spmv_od
bash scripts/prof.sh r01h C4 f64 0 coo_spmv
