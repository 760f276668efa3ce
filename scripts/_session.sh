OUT=gpurun_out/r02o; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or pdl or x_window" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -2 $OUT/pytest_q.txt
for dt in f64 f32; do for T in 8 16 32; do timeout 600 python scripts/ab.py C4 $dt --format coo "coo_T=$T" --baseline-opts "coo_T=$T" > $OUT/ab_C4_coo_${dt}_T$T.txt 2>&1; tail -1 $OUT/ab_C4_coo_${dt}_T$T.txt | cut -c1-110; done; done
for dt in f64 f32; do for T in 8 16 32; do timeout 600 python scripts/ab.py C3 $dt --format coo "coo_T=$T" --baseline-opts "coo_T=$T" > $OUT/ab_C3_coo_${dt}_T$T.txt 2>&1; tail -1 $OUT/ab_C3_coo_${dt}_T$T.txt | cut -c1-110; head -1 $OUT/ab_C3_coo_${dt}_T$T.txt | cut -c1-60; done; done
for dt in f64 f32; do timeout 600 python scripts/ab.py C4 $dt "coo_T=8" "coo_T=16" "coo_T=32" --baseline-opts "coo_T=8" > $OUT/ab_C4_hyb_$dt.txt 2>&1; cat $OUT/ab_C4_hyb_$dt.txt | cut -c1-130; done
for dt in f64 f32; do timeout 600 python scripts/ab.py C3 $dt "coo_T=8" "coo_T=16" --baseline-opts "coo_T=8" > $OUT/ab_C3_hyb_$dt.txt 2>&1; cat $OUT/ab_C3_hyb_$dt.txt | cut -c1-130; done
