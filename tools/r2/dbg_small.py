import sys, numpy as np
sys.path.insert(0, '.')
import gen, oracle
from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
from tests.gpu_util import dev
A = gen.random_rows(int(sys.argv[1]) if len(sys.argv) > 1 else 3000, seed=21)
p = SpGemmPlan(dev(A), dev(A)); info = p.setup()
print("setup", info.nprods, info.small_rows, info.bitmap_rows, info.long_rows, flush=True)
nnz = p.symbolic(); print("symbolic", nnz, flush=True)
C = p.numeric(); rp, col, val = C.numpy()
W, sc, _ = oracle.spgemm(A, A)
print("rp", np.array_equal(rp, W.rp), "col", np.array_equal(col, W.col))
