#!/bin/bash
# compute-sanitizer memcheck / racecheck / initcheck over the small GPU parity cases (gpurun)
OUT=${1:-gpurun_out/sanitize}; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
K="spmv_random and (tiny or ragged or long or all_empty) or instances or coo_intervals or single_long or inf or empty_matrix or forced or scatter_matches or value_index_instances"
for tool in memcheck racecheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -q -x -p no:cacheprovider -k "$K" > $OUT/$tool.txt 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" $OUT/$tool.txt | tail -3
done
