OUT=gpurun_out/r02h; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or instances or pdl or spmv_random or configs_full" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/pytest_q.txt
timeout 900 python scripts/ab.py C5 f32 "slice_h=64,ell_kernel=6" "slice_h=64,ell_kernel=7" "slice_h=64,ell_kernel=8" > $OUT/ab_C5_f32.txt 2>&1; cat $OUT/ab_C5_f32.txt
timeout 900 python scripts/ab.py C4 f64 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,pdl=2" "slice_h=64,coo_T=8" "slice_h=32,coo_T=32" --baseline-opts "coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt
timeout 900 python scripts/ab.py C4 f32 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,pdl=2" "slice_h=64,coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C4_f32.txt 2>&1; cat $OUT/ab_C4_f32.txt
timeout 900 python scripts/ab.py C3 f64 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,pdl=2" "slice_h=32,coo_T=16" --baseline-opts "coo_T=8" > $OUT/ab_C3_f64.txt 2>&1; cat $OUT/ab_C3_f64.txt
timeout 900 python scripts/ab.py C3 f32 "slice_h=32,coo_T=8" "slice_h=32,coo_T=8,pdl=2" --baseline-opts "coo_T=8" > $OUT/ab_C3_f32.txt 2>&1; cat $OUT/ab_C3_f32.txt
NCU="ncu --set full --clock-control none --import-source on"
timeout 600 $NCU -k regex:bro_ell_od -s 2 -c 1 -o $OUT/C4_ell python scripts/prof_one.py C4 f64 "slice_h=32,coo_T=8" > $OUT/ncu1.log 2>&1; echo "ncu1 rc=$?"
timeout 600 $NCU -k regex:coo_spmv -s 2 -c 1 -o $OUT/C4_coo python scripts/prof_one.py C4 f64 "slice_h=32,coo_T=8" > $OUT/ncu2.log 2>&1; echo "ncu2 rc=$?"
timeout 600 $NCU -k regex:bro_ell_od -s 2 -c 1 -o $OUT/C5_x7 python scripts/prof_one.py C5 f64 "slice_h=32,ell_kernel=7" > $OUT/ncu3.log 2>&1; echo "ncu3 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file $OUT/launches_C4.csv python scripts/prof_one.py C4 f64 "slice_h=32,coo_T=8" --launches 10 > /dev/null 2>&1; python scripts/launch_summary.py $OUT/launches_C4.csv
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file $OUT/launches_C3.csv python scripts/prof_one.py C3 f64 "slice_h=32,coo_T=8" --launches 10 > /dev/null 2>&1; python scripts/launch_summary.py $OUT/launches_C3.csv
