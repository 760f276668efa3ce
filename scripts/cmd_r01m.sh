OUT=gpurun_out/r01m; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
bash scripts/prof.sh r01m C4 f64 0 coo_spmv
bash scripts/prof.sh r01m C3 f64 0 bro_ell_spmv_od --flush-l2
