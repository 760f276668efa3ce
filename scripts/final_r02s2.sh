#!/bin/bash
# Round-2 session-2 evidence run (one gpurun call): full GPU suite, smoke,
# sanitizers, default bench line, every config/dtype (+ value-index and
# standalone COO lines), launch lists and ncu --set full captures.
OUT=${OUT:-gpurun_out/r03z}; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw,clocks_event_reasons.active --format=csv > $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail -30 $OUT/build.txt; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.txt
[ -n "$SANITIZE" ] && bash scripts/sanitize.sh $OUT/sanitizer  # compute-sanitizer is refused on this pool (profiles/r02/s2/final/sanitizer_refused.txt)
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cut -c1-300 $OUT/bench.json
summ() { python - "$1" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d["roofline"]; u=d["uncompressed"]; c=d["config"]
    print(f'  {c["workload"][:3]} {d["dtype"]} {c["format"]} h={c["slice_h"]} inst={c["ell_kernel"]} kern {r["kernel_ms"]*1e3:.1f}us {r["achieved"]:.0f}GB/s frac {r["frac"]:.3f} | {u["format"]} {u["kernel_ms"]*1e3:.1f}us x{u["kernel_ms"]/r["kernel_ms"]:.3f} | e2e {d["e2e"]["value"]:.1f} | clocks {d.get("clocks")}')
except Exception as e: print("  parse error", e)
PY
}
for wl in C1 C2 C3 C4 C5; do for dt in f64 f32; do
  fl=""; [ $wl = C1 -o $wl = C2 -o $wl = C3 ] && fl="--flush-l2"
  timeout 900 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline $fl > $OUT/bench_${wl}_${dt}.json 2>> $OUT/benchall.err; summ $OUT/bench_${wl}_${dt}.json
done; done
for wl in C1 C5; do for dt in f64 f32; do
  fl=""; [ $wl = C1 ] && fl="--flush-l2"
  timeout 900 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline --value-codec 1 $fl > $OUT/bench_${wl}_${dt}_vi.json 2>> $OUT/benchall.err; summ $OUT/bench_${wl}_${dt}_vi.json
done; done
for wl in C3 C4; do for dt in f64 f32; do
  fl=""; [ $wl = C3 ] && fl="--flush-l2"
  timeout 900 python bench.py --workload $wl --dtype $dt --steps 500 --no-cpu-baseline --format coo $fl > $OUT/bench_${wl}_${dt}_coo.json 2>> $OUT/benchall.err; summ $OUT/bench_${wl}_${dt}_coo.json
done; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $OUT/launches_C5.csv \
  python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/launches_bench.log 2>&1; echo "launches rc=$?"
python scripts/launch_summary.py $OUT/launches_C5.csv | tee $OUT/launches_C5_summary.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file $OUT/launches_C4.csv \
  python scripts/prof_one.py C4 f64 "" --launches 10 > /dev/null 2>&1; python scripts/launch_summary.py $OUT/launches_C4.csv | tee $OUT/launches_C4_summary.txt
for v in "C5 f64 slice_h=64" "C5 f32 slice_h=64" "C5 f64 value_codec=1" "C4 f64 slice_h=64" ; do
  set -- $v; tag=${1}_${2}_$(echo $3 | tr '=,' '__')
  timeout 900 ncu --set full --clock-control none --import-source on -s 3 -c 3 -o $OUT/full_$tag python scripts/prof_one.py $1 $2 "$3" > $OUT/ncu_$tag.log 2>&1; echo "ncu $tag rc=$?"
  python scripts/ncu_summary.py $OUT/full_$tag.ncu-rep 12 > $OUT/ncu_$tag.txt 2>&1; grep -E "Kernel Name|gpu__time|dram__bytes" $OUT/ncu_$tag.txt
done
