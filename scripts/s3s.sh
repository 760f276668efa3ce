#!/bin/bash
OUT=gpurun_out/s3s; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 600 python bench.py --steps 300 --warmup 10 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cut -c1-300 $OUT/bench.json
python -c "import json; d=json.load(open('$OUT/bench.json')); print(d['roofline']); print(d['gpu_launches'], d['clocks'])"
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/ref.json 2> $OUT/ref.err; echo "ref rc=$?"; cut -c1-300 $OUT/ref.json
