#!/bin/bash
# A/B kernel timing in one session: libbro.so (current) vs libbro_ab.so (another build), alternated
# usage: bash scripts/ab.sh TAG "bench args" [rounds]
TAG=$1; ARGS=$2; R=${3:-3}; OUT=gpurun_out/$TAG; mkdir -p $OUT
for r in $(seq 1 $R); do
  for lib in libbro.so libbro_ab.so; do
    BRO_LIB=$lib timeout 600 python bench.py $ARGS --no-cpu-baseline --no-e2e > $OUT/ab_${lib}_$r.json 2>>$OUT/ab.err
    python -c "import json; d=json.load(open('$OUT/ab_${lib}_$r.json')); print('$lib', $r, round(d['roofline']['kernel_ms']*1e3,1), 'us', round(d['roofline']['frac'],3), 'base', round(d['uncompressed']['kernel_ms']*1e3,1))"
  done
done
