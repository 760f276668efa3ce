OUT=gpurun_out/r02m; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
K="(spmv_random and (tiny or ragged or long or all_empty)) or (instances and float64) or coo_intervals or single_long or inf or empty_matrix or forced or pdl or scatter_matches"
for tool in memcheck racecheck initcheck; do
  timeout 1700 compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -q -x -p no:cacheprovider -k "$K" > $OUT/$tool.txt 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" $OUT/$tool.txt | tail -3
done
