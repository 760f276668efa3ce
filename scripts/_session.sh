OUT=gpurun_out/r02e; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
python -c "import sys; sys.path.insert(0,'scripts'); import ab_r1; ab_r1.build_r1()" > $OUT/build_r1.txt 2>&1 || echo r1 build failed
NCU="ncu --set full --clock-control none --import-source on"
timeout 600 $NCU -k regex:bro_ell_spmv_od -s 2 -c 1 -o $OUT/r1_C5_f64 python scripts/prof_one.py C5 f64 --r1 > $OUT/ncu1.log 2>&1; echo "r1 rc=$?"
timeout 600 $NCU -k regex:bro_ell_od -s 2 -c 1 -o $OUT/new_C5_f64_small python scripts/prof_one.py C5 f64 "slice_h=32,ell_kernel=3" > $OUT/ncu2.log 2>&1; echo "new rc=$?"
timeout 600 $NCU -k regex:bro_ell_od -s 2 -c 1 -o $OUT/new_C5_f64_x10 python scripts/prof_one.py C5 f64 "slice_h=64,ell_kernel=10" > $OUT/ncu3.log 2>&1; echo "x10 rc=$?"
timeout 600 $NCU -k regex:bro_ell_od -s 2 -c 1 -o $OUT/new_C5_f32_x6 python scripts/prof_one.py C5 f32 "slice_h=64,ell_kernel=6" > $OUT/ncu4.log 2>&1; echo "f32 x6 rc=$?"
timeout 600 $NCU -k regex:coo_spmv -s 2 -c 1 -o $OUT/coo_bro_C4 python scripts/prof_one.py C4 f64 "coo_T=8" --format coo > $OUT/ncu5.log 2>&1; echo "coo bro rc=$?"
timeout 600 $NCU -k regex:coo_spmv -s 2 -c 1 -o $OUT/coo_plain_C4 python scripts/prof_one.py C4 f64 "coo_T=8" --format coo --codec 0 > $OUT/ncu6.log 2>&1; echo "coo plain rc=$?"
ls -la $OUT
