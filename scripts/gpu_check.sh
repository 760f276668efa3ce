#!/bin/bash
# One gpurun call: build, GPU parity tests, smoke, bench, ncu launch list + full capture.
# usage: bash scripts/gpu_check.sh [tag] [what...]   (what: tests smoke bench ncu full)
TAG=${1:-r01}
shift || true
WHAT=${@:-tests smoke bench ncu full}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,clocks.mem,power.draw,clocks_event_reasons.active --format=csv >> $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; cat $OUT/build.txt; exit 1; }
for w in $WHAT; do
  case $w in
    tests)
      timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
      echo "pytest rc=$?"; tail -5 $OUT/pytest_gpu.txt ;;
    alltests)
      timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
      echo "pytest rc=$?"; tail -15 $OUT/pytest_gpu.txt ;;
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -3 $OUT/smoke.txt ;;
    bench)
      timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cat $OUT/bench.json; tail -3 $OUT/bench.err ;;
    bench_all)
      for wl in C1 C2 C3 C4; do
        for dt in f64 f32; do
          timeout 600 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline --flush-l2 > $OUT/bench_${wl}_${dt}.json 2>> $OUT/bench_all.err
          echo "$wl $dt rc=$?"; cut -c1-400 $OUT/bench_${wl}_${dt}.json
        done
      done ;;
    ncu)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
        --log-file $OUT/launches_C5.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.txt 2>&1
      echo "ncu launches rc=$?" ;;
    full)
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv -s 3 -c 1 \
        -o $OUT/prof_C5_bro_ell python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full.txt 2>&1
      echo "ncu full rc=$?"
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:^ell_spmv -s 3 -c 1 \
        -o $OUT/prof_C5_plain_ell python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full2.txt 2>&1
      echo "ncu full2 rc=$?" ;;
  esac
done
