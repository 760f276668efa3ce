bash scripts/sanitize.sh gpurun_out/r01w
python scripts/sweep.py gpurun_out/r01w "0" "C5:f32 C5:f64 C4:f32 C4:f64 C3:f64 C2:f64" 2>&1
