bash scripts/sanitize.sh gpurun_out/r01r
python scripts/sweep.py gpurun_out/r01r "0" "C5:f64 C5:f32 C4:f64 C4:f32 C2:f64 C3:f64" 2>&1
