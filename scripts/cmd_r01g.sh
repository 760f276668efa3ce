OUT=gpurun_out/r01g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cat $OUT/bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C5.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "launches rc=$?"
bash scripts/prof.sh r01g C5 f64 0 bro_ell_spmv_od
bash scripts/prof.sh r01g C5 f32 0 bro_ell_spmv_od
bash scripts/prof.sh r01g C3 f64 0 coo_spmv --flush-l2
bash scripts/prof.sh r01g C4 f64 0 coo_spmv
