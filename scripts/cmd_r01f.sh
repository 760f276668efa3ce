bash scripts/run_sweep.sh r01f "0" "C5:f64:0,1,2,3 C5:f32:0,1,2,3 C2:f64:0,1 C4:f64:0,1 C4:f32:0 C2:f32:0 C3:f64:0 C1:f64:0" "spmv_random or vec_words or decode or config5_full or single_long or inf or config4 or row_blocks"
bash scripts/prof.sh r01f C5 f64 0 bro_ell_spmv_pf
bash scripts/prof.sh r01f C5 f32 0 bro_ell_spmv_pf
