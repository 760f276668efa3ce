OUT=gpurun_out/r02n; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "x_window or instances" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/pytest_q.txt
for dt in f64 f32; do timeout 600 python scripts/ab.py C2 $dt "x_stage=0" "x_stage=2" > $OUT/ab_C2_$dt.txt 2>&1; cat $OUT/ab_C2_$dt.txt; done
for dt in f64 f32; do timeout 600 python scripts/ab.py C1 $dt "x_stage=0" "x_stage=2" > $OUT/ab_C1_$dt.txt 2>&1; cat $OUT/ab_C1_$dt.txt; done
timeout 1500 python scripts/bar_eval.py --gpu --configs 4,2 --out $OUT/bar_eval.json > $OUT/bar_eval.txt 2>&1; cat $OUT/bar_eval.txt | tail -12
