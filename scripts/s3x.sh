#!/bin/bash
OUT=gpurun_out/s3x; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_instances.py tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -k "config5 or stencil or scatter or row_block or tiny or host" > $OUT/pytest.txt 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python -c "import json; d=json.load(open('$OUT/bench.json')); r=d['roofline']; print(d['value'], r['kernel_ms'], r['frac'], d['uncompressed']['speedup_bro'], d['e2e']['value'], d['clocks'])"
timeout 600 python bench.py --dtype f32 --steps 500 --no-cpu-baseline > $OUT/bench_f32.json 2>> $OUT/bench.err
python -c "import json; d=json.load(open('$OUT/bench_f32.json')); r=d['roofline']; print(d['value'], r['kernel_ms'], r['frac'], d['uncompressed']['speedup_bro'], d['e2e']['value'], d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $OUT/launches_C5.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo "ncu rc=$?"
python scripts/launch_summary.py $OUT/launches_C5.csv
