OUT=gpurun_out/r01n; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || exit 1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 50 --warmup 3 --dist-backend gloo --no-cpu-baseline > $OUT/bench_n2_gloo.json 2> $OUT/bench_n2_gloo.err; echo "n2 rc=$?"; cat $OUT/bench_n2_gloo.json; tail -5 $OUT/bench_n2_gloo.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 1 --steps 200 --warmup 3 --no-cpu-baseline > $OUT/bench_n1_torchrun.json 2> $OUT/bench_n1.err; echo "n1 torchrun rc=$?"; cut -c1-300 $OUT/bench_n1_torchrun.json
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/bench_ref.json 2> $OUT/bench_ref.err; echo "ref rc=$?"; cat $OUT/bench_ref.json
