"""B200-native TileSpMV hot path (Niu et al., IPDPS 2021): fp64 y = A x over
16x16 sparse tiles in seven formats with a CSR remainder.

    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    A = TiledMatrix.from_csr(rowptr, colidx, val, m, n)   # CUDA tensors
    y = A.run(x)

The compute lives in libtilespmv.so (csrc/, C ABI in include/tilespmv.h).
"""
from .tilespmv import (EXPORTED_SYMBOLS, FORMATS, MODES, TiledMatrix, TileSpMVError,  # noqa: F401
                       load)
