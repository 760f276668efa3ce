#!/bin/bash
OUT=gpurun_out/s3q; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bro_ell_spmv -s 3 -c 1 \
  -o $OUT/prof_C2_f64 python bench.py --workload C2 --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --flush-l2 > $OUT/ncu_c2.txt 2>&1
echo "ncu C2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"bro_ell_spmv|coo_spmv|coo_fixup" -s 3 -c 3 \
  -o $OUT/prof_C3_f64 python bench.py --workload C3 --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --flush-l2 > $OUT/ncu_c3.txt 2>&1
echo "ncu C3 rc=$?"
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29535 \
  bench.py --gpus 2 --workload C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --dist-backend gloo \
  > $OUT/bench_gloo2_C5_auto.json 2> $OUT/bench_gloo2_C5_auto.err
echo "gloo2 C5 rc=$?"; python -c "import json; d=json.load(open('$OUT/bench_gloo2_C5_auto.json')); print(d['exchange'], d['gpu_launches'])"; tail -3 $OUT/bench_gloo2_C5_auto.err
