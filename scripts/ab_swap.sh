# A/B of two builds of libbro.so in one gpurun session (same box, back to back):
#   bash scripts/ab_swap.sh OUTDIR "ab.py args" [rounds]   (scratch_ab/libbro_{old,new}.so)
OUT=$1; ARGS=$2; R=${3:-2}; mkdir -p $OUT
L=paper_conf_sc_tangtrwckgtw13_b200/libbro.so
for r in $(seq $R); do for v in old new; do
  cp scratch_ab/libbro_$v.so $L
  echo "== $v (round $r)" >> $OUT/ab.txt
  timeout 900 python scripts/ab.py $ARGS >> $OUT/ab.txt 2>&1
done; done
cp scratch_ab/libbro_new.so $L
