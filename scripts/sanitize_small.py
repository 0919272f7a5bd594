"""Small SpMV runs for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): every format, both modes, edge shapes; each checked against the
oracle.  Usage: compute-sanitizer --tool memcheck python scripts/sanitize_small.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from oracle import oracle as O  # noqa: E402
from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix  # noqa: E402
from synthetic import gen  # noqa: E402

mats = [gen.make(n)[0] for n in ("lap2d_37x29", "mixed_small", "rmat12", "stencil27_21", "fem_small")]
mats += [gen.random_sparse(17, 33, 0.3, seed=1), gen.random_sparse(1, 1, 1.0),
         gen.random_sparse(70, 70, 0.95, seed=4, empty_rows=range(16, 32))]
bad = 0
for A in mats:
    x = gen.dense_x(A.n, 101)
    yref, absy = O.spmv(A, x)
    for mode in ("ADPT", "DEFERRED"):
        for kernel in ("SM_QUEUE", "DENSE_ROWS", "GATHER"):
            M = TiledMatrix.from_host_csr(A, mode=mode, kernel=kernel)
            y = M.run(torch.from_numpy(x).cuda()).cpu().numpy()
            ok = np.all(np.abs(y - yref) <= 1e-12 * absy + 1e-300)
            bad += not ok
            print(A.name, mode, kernel, "ok" if ok else "MISMATCH", flush=True)
            M.close()
torch.cuda.synchronize()
print("sanitize_small done, mismatches:", bad)
sys.exit(1 if bad else 0)
