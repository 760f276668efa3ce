#!/bin/bash
TAG=s3c; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; tail $OUT/build.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -rs -k "world2 or single" > $OUT/pytest_dist.txt 2>&1
echo "pytest rc=$?"; tail -8 $OUT/pytest_dist.txt
for ex in overlap; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 \
    bench.py --gpus 2 --workload C2 --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --dist-backend gloo --exchange $ex \
    > $OUT/bench_gloo_C2_$ex.json 2> $OUT/bench_gloo_C2_$ex.err
  echo "gloo C2 $ex rc=$?"; python -c "import json; d=json.load(open('$OUT/bench_gloo_C2_$ex.json')); print(d['value'], d['exchange'])" ; tail -3 $OUT/bench_gloo_C2_$ex.err
done
bash scripts/ab.sh $TAG "--workload C5 --steps 300 --warmup 10" 2
