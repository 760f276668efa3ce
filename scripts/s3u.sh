#!/bin/bash
OUT=gpurun_out/s3u; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_instances.py tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "host or pipelined" > $OUT/pytest.txt 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest.txt
for wl in C1 C2 C5; do
timeout 600 python bench.py --workload $wl --steps 200 --warmup 5 --no-cpu-baseline > $OUT/bench_$wl.json 2>> $OUT/bench.err
python -c "import json; d=json.load(open('$OUT/bench_$wl.json')); print('$wl', d['e2e']['value'], d['e2e']['ms_per_step'])"
done
