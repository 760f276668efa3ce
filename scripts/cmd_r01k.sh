bash scripts/run_sweep.sh r01k "0" "C5:f64:0,1 C5:f32:0,1 C4:f64:0,1 C4:f32:0 C3:f64:0,1 C2:f64:0,1" "spmv_random or decode or single_long or config4 or determin"
