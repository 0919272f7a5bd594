"""A/B helper (scripts/gpu_ab_lib.sh): y of a few configs with the loaded libtilespmv.so, saved to an .npz for a bitwise old/new comparison."""
import sys, numpy as np, torch
sys.path.insert(0, '.')
from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
from synthetic import gen
out = {}
for name in ("rmat12", "mixed_small", "stencil27_40", "rmat20", "mixed"):
    A, x = gen.make(name)
    for mode in ("DEFERRED", "ADPT"):
        M = TiledMatrix.from_host_csr(A, mode=mode, device=torch.device("cuda", 0))
        out[f"{name}_{mode}"] = M.run(torch.from_numpy(x).cuda()).cpu().numpy()
        M.close()
np.savez(sys.argv[1], **out)
