#!/bin/bash
# usage: bash scripts/run_sweep.sh TAG "variants" "cases" [pytest -k expr]
TAG=$1; VARS=$2; CASES=$3; KEXPR=${4:-}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { cat $OUT/build.txt; exit 1; }
if [ -n "$KEXPR" ]; then
  timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "$KEXPR" > $OUT/pytest.txt 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest.txt
fi
python scripts/sweep.py $OUT "$VARS" "$CASES" 2>&1
