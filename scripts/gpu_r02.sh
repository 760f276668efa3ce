#!/bin/bash
# One gpurun session of round 2: build, then the steps named on the command line.
#   bash scripts/gpu_r02.sh TAG step...    steps: tests quick smoke bench benchall ab_* launches full_C5 sanitize
TAG=${1:-r02}; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw,clocks_event_reasons.active --format=csv > $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build.txt; exit 1; }
for w in "$@"; do
  case $w in
    tests) timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu.txt 2>&1
           echo "pytest rc=$?"; tail -6 $OUT/pytest_gpu.txt ;;
    quick) timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x \
             -k "spmv_random or instances or coo_intervals or forced or inf or vector or empty or single" > $OUT/pytest_quick.txt 2>&1
           echo "quick rc=$?"; tail -6 $OUT/pytest_quick.txt ;;
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke.txt ;;
    bench) timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cut -c1-1500 $OUT/bench.json; tail -3 $OUT/bench.err ;;
    benchall)
      for wl in C1 C2 C3 C4 C5; do for dt in f64 f32; do
        fl=""; [ $wl = C1 -o $wl = C2 -o $wl = C3 ] && fl="--flush-l2"
        timeout 900 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/benchall.err
        echo "$wl $dt rc=$?"; python - $OUT/bench_${wl}_${dt}.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d["roofline"]; u=d["uncompressed"]
    print(f'  {d["config"]["workload"][:3]} {d["dtype"]} {d["config"]["format"]} h={d["config"]["slice_h"]} T={d["config"]["coo_T"]} kern {r["kernel_ms"]*1e3:.1f}us {r["achieved"]:.0f}GB/s frac {r["frac"]:.3f} | base {u["kernel_ms"]*1e3:.1f}us x{u["kernel_ms"]/r["kernel_ms"]:.3f} | e2e {d["e2e"]["value"]:.1f}')
except Exception as e: print("  parse error", e)
PY
      done; done ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $OUT/launches_C5.csv \
                python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/launches_bench.log 2>&1
              echo "launches rc=$?"; python scripts/launch_summary.py $OUT/launches_C5.csv ;;
    sanitize) bash scripts/sanitize.sh $OUT/sanitizer ;;
    *) echo "unknown step $w" ;;
  esac
done
