bash scripts/sanitize.sh gpurun_out/r01s
python scripts/sweep.py gpurun_out/r01s "0" "C5:f32 C5:f64 C4:f32 C2:f32" 2>&1
