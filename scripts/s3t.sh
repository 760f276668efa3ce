#!/bin/bash
OUT=gpurun_out/s3t; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_instances.py tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "host or pipelined" > $OUT/pytest.txt 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest.txt
for k in 1 8 16; do
BRO_E2E_CHUNKS=$k timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu-baseline > $OUT/bench_k$k.json 2> $OUT/bench.err
python -c "import json; d=json.load(open('$OUT/bench_k$k.json')); print('K=$k', d['e2e']['value'], d['e2e']['ms_per_step'], d['roofline']['kernel_ms'])"
done
BRO_E2E_CHUNKS=8 timeout 600 python bench.py --workload C2 --steps 100 --warmup 5 --no-cpu-baseline > $OUT/bench_c2.json 2>> $OUT/bench.err
python -c "import json; d=json.load(open('$OUT/bench_c2.json')); print('C2', d['e2e']['value'], d['e2e']['ms_per_step'])"
