#!/bin/bash
OUT=gpurun_out/s3j; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { echo BUILD FAILED; exit 1; }
V="BRO_ELL_SMALLWIN=0 BRO_ELL_SMALLWIN=1 BRO_ELL_SMALLWIN=0 BRO_ELL_SMALLWIN=1"
for c in "C5 f64" "C5 f32"; do
  timeout 900 python scripts/sweep_env.py $c ell "$V" 300 2>&1 | tee -a $OUT/sweep.txt | grep -v Warn
done
python - <<'PY' >> $OUT/sweep.txt
import numpy as np, sys
sys.path.insert(0,'.')
import bench, paper_conf_sc_tangtrwckgtw13_b200 as P
for wl in ("C2","C3","C4","C5"):
    A,fmt = bench.load_workload(wl, np.float64, P)
    M = P.BroMatrix(A, fmt=fmt, codec=1, device=0)
    print(wl, "n_slices", M.info["n_slices"])
PY
tail -4 $OUT/sweep.txt
