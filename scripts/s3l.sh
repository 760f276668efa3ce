#!/bin/bash
OUT=gpurun_out/s3l; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_instances.py -m gpu -q -p no:cacheprovider -k "tiny or stencil" > $OUT/pytest_inst.txt 2>&1
echo "pytest inst rc=$?"; tail -3 $OUT/pytest_inst.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "coo or hyb or determ or config3 or config4" > $OUT/pytest_par.txt 2>&1
echo "pytest parity rc=$?"; tail -3 $OUT/pytest_par.txt
V="BRO_ELL_TINY=0 BRO_ELL_TINY=1 BRO_ELL_TINY=2 BRO_ELL_TINY=0 BRO_ELL_TINY=1 BRO_ELL_TINY=2"
for c in "C3 f64" "C3 f32"; do
  timeout 900 python scripts/sweep_env.py $c hyb,coo "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file $OUT/launches_C3.csv \
  python bench.py --workload C3 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "ncu rc=$?"
python scripts/launch_summary.py $OUT/launches_C3.csv
