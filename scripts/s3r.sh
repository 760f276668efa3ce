#!/bin/bash
OUT=gpurun_out/s3r; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
for dt in f32 f64; do for vw in 1 2 4; do
  timeout 600 python bench.py --workload C5 --dtype $dt --vec-words $vw --steps 300 --warmup 10 --no-cpu-baseline --no-e2e > $OUT/b_${dt}_v$vw.json 2>/dev/null
  python -c "import json; d=json.load(open('$OUT/b_${dt}_v$vw.json')); print('$dt V=$vw', round(d['roofline']['kernel_ms']*1e3,1), 'us', round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done
