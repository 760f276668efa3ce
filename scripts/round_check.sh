#!/bin/bash
# One gpurun call: build, full GPU tests, smoke, default bench, all-config benches,
# BAR ordering evaluation, ncu launch list of the default bench.
# usage: bash scripts/round_check.sh TAG [what...]  (what: tests smoke bench all bar ncu)
TAG=${1:-r01}; shift || true
WHAT=${@:-tests smoke bench all bar ncu}
OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail $OUT/build.txt; exit 1; }
for w in $WHAT; do
  case $w in
    tests) timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
           echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.txt ;;
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?" ;;
    bench) timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cat $OUT/bench.json ;;
    all) for wl in C1 C2 C3 C4 C5; do for dt in f64 f32; do
           fl=""; [ $wl = C1 -o $wl = C2 -o $wl = C3 ] && fl="--flush-l2"
           timeout 600 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/bench_all.err
           echo "$wl $dt rc=$?"; done; done
         for wl in C3 C4; do timeout 600 python bench.py --workload $wl --format coo --steps 300 --no-cpu-baseline --no-e2e \
           $( [ $wl = C3 ] && echo --flush-l2 ) > $OUT/bench_${wl}_coo.json 2>> $OUT/bench_all.err; echo "$wl coo rc=$?"; done ;;
    bar) timeout 1200 python scripts/bar_eval.py --gpu --out $OUT/bar_eval.json > $OUT/bar_eval.txt 2>&1; echo "bar rc=$?"; cat $OUT/bar_eval.txt ;;
    ncu) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
           --log-file $OUT/launches_C5.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.txt 2>&1
         echo "ncu launches rc=$?" ;;
  esac
done
