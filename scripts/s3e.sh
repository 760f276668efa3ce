#!/bin/bash
OUT=gpurun_out/s3e; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
bash scripts/ab.sh s3e "--workload C5 --steps 300 --warmup 10" 2
bash scripts/ab.sh s3e "--workload C5 --dtype f32 --steps 300 --warmup 10" 1
bash scripts/ab.sh s3e "--workload C4 --steps 300 --warmup 10" 1
