python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python scripts/sweep.py gpurun_out/r01x "0" "C5:f32 C5:f64 C4:f32" 2>&1
