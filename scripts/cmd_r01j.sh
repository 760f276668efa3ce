OUT=gpurun_out/r01j; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
timeout 900 python scripts/eta_sweep.py $OUT/eta_sweep.json 2>&1 | tee $OUT/eta_sweep.txt | head -60
python scripts/sweep.py $OUT "0" "C1:f64 C2:f64 C2:f32 C3:f64 C3:f32 C4:f64 C4:f32 C5:f64 C5:f32" 2>&1
