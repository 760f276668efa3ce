OUT=gpurun_out/r02t; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1 || { tail $OUT/build.txt; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -q -p no:cacheprovider -x -k "coo_intervals or pdl or spmv_random or single or config4 or configs_full or scatter or deterministic or side_stream" > $OUT/pytest_q.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/pytest_q.txt
timeout 600 python scripts/ab.py C4 f64 "coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C4_f64.txt 2>&1; cat $OUT/ab_C4_f64.txt | cut -c1-120
timeout 600 python scripts/ab.py C4 f32 "coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C4_f32.txt 2>&1; cat $OUT/ab_C4_f32.txt | cut -c1-120
timeout 600 python scripts/ab.py C3 f64 "coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C3_f64.txt 2>&1; cat $OUT/ab_C3_f64.txt | cut -c1-120
timeout 600 python scripts/ab.py C3 f32 "coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_C3_f32.txt 2>&1; cat $OUT/ab_C3_f32.txt | cut -c1-120
for wl in C3 C4; do for f in hyb coo; do timeout 600 python scripts/ab.py $wl f64 --format $f "coo_T=8" --baseline-opts "coo_T=8" > $OUT/ab_${wl}_${f}.txt 2>&1; tail -2 $OUT/ab_${wl}_${f}.txt | cut -c1-120; done; done
for wl in C3 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file $OUT/launches_$wl.csv python scripts/prof_one.py $wl f64 --launches 10 > /dev/null 2>&1; python scripts/launch_summary.py $OUT/launches_$wl.csv
done
python - <<'PY'
# CUDA graph replay of a HYB handle: the look-back's epoch lives in device memory
import sys; sys.path.insert(0,'.')
import numpy as np, torch
import paper_conf_sc_tangtrwckgtw13_b200 as P
from gen import random_csr, make_x
from oracle import spmv
A = random_csr(20000, 20000, 3, max_len=8, long_frac=0.01, long_len=3000)
M = P.BroMatrix(A, fmt="hyb", device=0)
x = torch.from_numpy(make_x(A.n, 1)).cuda(); y = torch.empty(A.m, dtype=torch.float64, device="cuda")
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    M.spmv(x, y, s)
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=s):
    M.spmv(x, y, s)
ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, make_x(A.n, 1))
ok = True
for k in range(20):
    y.zero_(); g.replay(); torch.cuda.synchronize()
    ok &= bool(spmv.within_tolerance(y.cpu().numpy(), ref, S, 1e-12)[0].all())
print("graph replays ok:", ok)
PY
