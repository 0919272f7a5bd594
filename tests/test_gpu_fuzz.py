"""GPU fuzz parity over tile-row shapes: seeded random matrices built tile by
tile so that every CSR-tile row-length profile the kernels special-case occurs
(equal rows of every length 1..16 laid end to end -- the lane-rotated reads of
pair extents 6..8 and 13..16 -- and ragged rows of 0..16 entries), mixed with
sparse COO-sized tiles, dense tiles and remainder-heavy rows, on ragged
m, n.  Each run is checked against the oracle SpMV within the north_star
tolerance (fp64) and for run-to-run bitwise determinism, in every mode
 on both SpMV kernels."""
import numpy as np
import pytest

from oracle import oracle as O
from synthetic import gen

from test_gpu_parity import assert_spmv_close


def tile_profile_matrix(m, n, seed, profile):
    """Input generator only (no SpMV arithmetic): a CSR whose 16x16 tiles
    follow `profile` ("equal", "ragged" or "blend")."""
    rng = np.random.default_rng(seed)
    tm, tn = (m + 15) // 16, (n + 15) // 16
    rows, cols = [], []
    for I in range(tm):
        for J in range(tn):
            u = rng.random()
            if u < 0.35:
                continue
            if profile == "equal" or (profile == "blend" and u < 0.6):
                L = int(rng.integers(1, 17))
                lens = np.full(16, L)
            elif profile == "ragged" or u < 0.8:
                lens = rng.integers(0, 17, size=16)
            else:  # COO-sized tile or a dense tile
                lens = rng.integers(0, 2, size=16) if u < 0.9 else np.full(16, 16)
            for r in range(16):
                cs = rng.choice(16, size=int(lens[r]), replace=False)
                rows.extend([16 * I + r] * len(cs))
                cols.extend((16 * J + cs).tolist())
    # a few long rows crossing every tile column (remainder / split rows)
    for r in rng.choice(m, size=min(3, m), replace=False):
        cs = rng.choice(n, size=min(n, 40 + int(rng.integers(0, 200))), replace=False)
        rows.extend([int(r)] * len(cs))
        cols.extend(cs.tolist())
    rows, cols = np.asarray(rows, np.int64), np.asarray(cols, np.int64)
    keep = (rows < m) & (cols < n)
    return gen.csr_from_coo(m, n, rows[keep], cols[keep], seed=seed + 1, name=f"{profile}{seed}")


CASES = [(128, 128, 0, "equal"), (125, 131, 1, "equal"), (200, 96, 2, "ragged"),
         (97, 203, 3, "ragged"), (160, 160, 4, "blend"), (143, 177, 5, "blend")]


@pytest.mark.gpu
@pytest.mark.parametrize("kernel", ["SM_QUEUE", "DENSE_ROWS", "GATHER"])
def test_tile_profile_fuzz(cuda_device, kernel):
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    for (m, n, seed, profile) in CASES:
        A = tile_profile_matrix(m, n, seed, profile)
        x = gen.dense_x(n, 7 + seed)
        yref, absy = O.spmv(A, x)
        xd = torch.from_numpy(x).to(cuda_device)
        for mode in ("ADPT", "DEFERRED", "FORCE_CSR", "BYTES"):
            M = TiledMatrix.from_host_csr(A, mode=mode, device=cuda_device, kernel=kernel)
            y1 = M.run(xd).cpu().numpy()
            y2 = M.run(xd).cpu().numpy()
            assert_spmv_close(y1, yref, absy, f"{profile}{seed}/{mode}/{kernel}")
            assert np.array_equal(y1.view(np.uint64), y2.view(np.uint64))
            M.close()


def test_tile_profile_generator_covers_profiles():
    """Host-only check of the generator: the equal profile yields tiles whose
    rows all have one length, and lengths 6..8 and 13..16 all occur."""
    A = tile_profile_matrix(256, 256, 11, "equal")
    seen = set()
    for I in range(16):
        for J in range(16):
            lens = []
            for r in range(16 * I, 16 * I + 16):
                c = A.colidx[A.rowptr[r]:A.rowptr[r + 1]]
                lens.append(int(np.count_nonzero((c >> 4) == J)))
            if any(lens) and len(set(lens)) == 1:
                seen.add(lens[0])
    assert {6, 7, 8, 13, 14, 15, 16} <= seen
