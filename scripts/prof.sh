#!/bin/bash
# usage: bash scripts/prof.sh TAG WORKLOAD DTYPE VARIANT KERNEL_REGEX [extra bench args]
TAG=$1; WL=$2; DT=$3; VAR=$4; KRE=$5; shift 5
OUT=gpurun_out/$TAG; mkdir -p $OUT
BRO_ELL_VARIANT=$VAR timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KRE" -s 3 -c 1 \
  -o $OUT/prof_${WL}_${DT}_v${VAR} python bench.py --workload $WL --dtype $DT --steps 6 --warmup 3 \
  --no-cpu-baseline --no-e2e "$@" > $OUT/prof_${WL}_${DT}_v${VAR}.txt 2>&1
echo "prof $WL $DT v$VAR rc=$?"
