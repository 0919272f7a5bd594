"""Pins for the reference tiler (§III.B, §III.D):
hand-built tiles at every selection boundary with hand-written payload bytes,
the HYB width scan against brute force, closed-form tile counts of the
structured configs, and the decode round trip.  CPU only."""
import itertools
import json
import os
import struct

import numpy as np
import pytest

from oracle import oracle as O
from synthetic import gen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
CSR, COO, ELL, HYB, DNS, DNSROW, DNSCOL = range(7)


def masks_from_lens(lens, rotate=True):
    """Row r gets lens[r] columns, rotated by r so that no two rows of equal
    length share a mask (avoids accidental DnsCol tiles)."""
    out = []
    for r, L in enumerate(lens):
        m = (1 << L) - 1
        if rotate:
            s = r % 16
            m = ((m << s) | (m >> (16 - s))) & 0xFFFF
        out.append(m)
    return out


def one_tile(entries, m=16, n=16, I=0, J=0):
    """entries: list of (r, c, v) inside tile (I, J)."""
    rows = [16 * I + r for r, _, _ in entries]
    cols = [16 * J + c for _, c, _ in entries]
    vals = [v for _, _, v in entries]
    return gen.csr_from_coo(m, n, rows, cols, vals=vals)


def f64(*vals):
    return b"".join(struct.pack("<d", v) for v in vals)


def pad16(b):
    return b + b"\0" * ((-len(b)) % 16)


def golden():
    with open(os.path.join(GOLDEN, "paper_constants.json")) as f:
        return json.load(f)


# --------------------------------------------------------------------------
# selection rules at every boundary
# --------------------------------------------------------------------------

def test_paper_constants_fixture():
    g = golden()
    assert g["tile"] == 16 and g["coo_below"] == 12 and g["dns_at_least"] == 128
    assert g["te"] == 0.2 and g["th"] == 1.0


@pytest.mark.parametrize("lens,fmt,aux", [
    ([1] * 11 + [0] * 5, COO, 0),                 # nnz 11 < 12
    ([1] * 12 + [0] * 4, CSR, 0),                 # nnz 12: CV = 0.577 -> CSR
    ([16] * 7 + [15] + [0] * 8, HYB, 0),          # nnz 127: not Dns; CV > 1
    ([16] * 8 + [0] * 8, DNS, 0),                 # nnz 128 -> Dns
    ([8] * 16, DNS, 0),                           # nnz 128, no full rows
    ([2] * 8 + [3] * 8, ELL, 3),                  # CV = 0.2 exactly -> ELL (closed)
    ([2] * 8 + [3] * 7 + [4], CSR, 0),            # CV = 0.243 -> CSR
    ([2] * 8 + [0] * 8, CSR, 0),                  # CV = 1.0 exactly -> CSR (open)
    ([0] * 8 + [2] + [3] * 7, HYB, 0),            # CV = 1.013 -> HYB, w = min = 0
    ([2] + [3] * 6 + [2, 1] + [0] * 7, CSR, 0),   # CV = 0.975 -> CSR
    ([3] * 7 + [2, 1] + [0] * 7, CSR, 0),         # CV = 0.972 -> CSR
    ([15, 15] + [1] * 14, HYB, 1),                # mixed-config HYB, w = 1
    ([1] * 15 + [16], HYB, 1),
    ([7] * 16, ELL, 7),                           # CV = 0
    ([1] * 16, ELL, 1),                           # Fig. 3 ELL: width 1
])
def test_select_rules(lens, fmt, aux):
    assert O.select(masks_from_lens(lens)) == (fmt, aux)


@pytest.mark.parametrize("k", range(1, 8))
def test_dense_rows_and_cols(k):
    full_rows = [0xFFFF if r < k else 0 for r in range(16)]
    assert O.select(full_rows) == (DNSROW, k)
    cols = (1 << k) - 1
    assert O.select([cols << 3] * 16) == (DNSCOL, k)
    if k == 7:  # 8 full rows / cols = 128 entries -> Dns
        assert O.select([0xFFFF] * 8 + [0] * 8) == (DNS, 0)
        assert O.select([0xFF] * 16) == (DNS, 0)


def test_force_csr():
    assert O.select([0xFFFF] * 16, force_csr=True) == (CSR, 0)
    assert O.select([1] + [0] * 15, force_csr=True) == (CSR, 0)


def _partitions(n, maxparts, maxval):
    if n == 0:
        yield []
        return
    if maxparts == 0:
        return
    for first in range(min(n, maxval), 0, -1):
        for rest in _partitions(n - first, maxparts - 1, first):
            yield [first] + rest


def test_coo_clause_is_implied():
    """Reading R4: any tile with < 12 entries has CV > te, i.e. "distributed
    not evenly among the rows" holds automatically."""
    for n in range(1, 12):
        for part in _partitions(n, 16, 16):
            lens = part + [0] * (16 - len(part))
            D = sum((16 * L - n) ** 2 for L in lens)
            assert 25 * D > 16 * n * n, (n, part)


def _hyb_mem(lens, w):
    return 16 * w * 8.5 + sum(max(0, L - w) * 9 for L in lens)


def test_hyb_width_scan_bruteforce():
    """P:105 scan vs brute force argmin (ties -> larger width) vs min(len)."""
    rng = np.random.default_rng(0)
    cases = [[1] * 15 + [16], [15, 15] + [1] * 14, [0] + [5] * 15]
    for _ in range(3000):
        kind = rng.integers(3)
        if kind == 0:
            lens = rng.integers(0, 17, 16)
        elif kind == 1:
            lens = np.minimum(16, rng.geometric(0.3, 16))
        else:
            lens = np.full(16, rng.integers(0, 17)); lens[rng.integers(16)] = rng.integers(0, 17)
        cases.append([int(v) for v in lens])
    for lens in cases:
        mems = [(_hyb_mem(lens, w), -w) for w in range(max(lens) + 1)]
        best = -min(mems)[1]
        assert O.hyb_width(lens) == best == min(lens), lens


# --------------------------------------------------------------------------
# level-2 payload bytes, hand-written per format
# --------------------------------------------------------------------------

def test_csr_payload_bytes():
    # rows 0-7: columns r and r+8; rows 8-15: column 23-r (n = 24, CV = 0.333)
    ents = []
    for r in range(8):
        ents += [(r, r, 0.0), (r, r + 8, 0.0)]
    for r in range(8, 16):
        ents.append((r, 23 - r, 0.0))
    ents = [(r, c, float(k + 1)) for k, (r, c, _) in enumerate(ents)]
    T = O.tile(one_tile(ents), "ADPT")
    assert T.numtile == 1 and T.tileFmt[0] == CSR and T.tileNnz[1] == 24
    rowptr = bytes([2 * r for r in range(8)] + [16 + r for r in range(8)])
    nib = bytes([0x80, 0x91, 0xA2, 0xB3, 0xC4, 0xD5, 0xE6, 0xF7, 0xEF, 0xCD, 0xAB, 0x89])
    expect = pad16(f64(*range(1, 25)) + rowptr + nib)
    assert len(expect) == 224
    assert T.payload.tobytes() == expect
    assert list(T.tileOff) == [0, 14]


def test_coo_payload_bytes():
    # Fig. 3's COO tile holds two entries
    T = O.tile(one_tile([(3, 5, 1.5), (10, 0, -2.0)]), "ADPT")
    assert T.tileFmt[0] == COO
    assert T.payload.tobytes() == pad16(f64(1.5, -2.0) + bytes([0x35, 0xA0]))
    Td = O.tile(one_tile([(3, 5, 1.5), (10, 0, -2.0)]), "DEFERRED")
    assert Td.numtile == 0 and Td.rem_nnz == 2
    assert list(Td.remRowPtr) == [0] * 4 + [1] * 7 + [2] * 6
    assert list(Td.remCol) == [5, 0] and list(Td.remVal) == [1.5, -2.0]


def test_ell_width1_payload_bytes():
    # one entry per row -> ELL, tilewidth 1 (Fig. 3 yellow tile)
    cols = [(5 * r) % 16 for r in range(16)]
    T = O.tile(one_tile([(r, cols[r], r + 0.25) for r in range(16)]), "ADPT")
    assert (T.tileFmt[0], T.tileAux[0]) == (ELL, 1)
    nib = bytes([cols[2 * j] | (cols[2 * j + 1] << 4) for j in range(8)])
    assert T.payload.tobytes() == pad16(f64(*[r + 0.25 for r in range(16)]) + nib)


def test_ell_pads_payload_bytes():
    # rows 0-7 hold columns {r, r+1}, rows 8-15 hold {0, 4, 9}: CV = 0.2 -> ELL w=3
    ents = []
    for r in range(16):
        cs = [r % 15, r % 15 + 1] if r < 8 else [0, 4, 9]
        ents += [(r, c, 100.0 * r + c) for c in cs]
    T = O.tile(one_tile(ents), "ADPT")
    assert (T.tileFmt[0], T.tileAux[0]) == (ELL, 3)
    vals, cols = [0.0] * 48, [0] * 48
    for r in range(16):
        cs = sorted(c for (rr, c, _) in ents if rr == r)
        for k, c in enumerate(cs):
            vals[16 * k + r] = 100.0 * r + c
            cols[16 * k + r] = c
    nib = bytes([cols[2 * j] | (cols[2 * j + 1] << 4) for j in range(24)])
    assert T.payload.tobytes() == pad16(f64(*vals) + nib)
    assert len(T.payload) == 416


def test_hyb_payload_bytes_and_extraction():
    # rows 0-14: column r; row 15 full -> CV > 1, HYB with w = min len = 1
    ents = [(r, r, float(r + 1)) for r in range(15)] + [(15, c, -float(c + 1)) for c in range(16)]
    A = one_tile(ents)
    T = O.tile(A, "ADPT")
    assert (T.tileFmt[0], T.tileAux[0]) == (HYB, 1)
    ell_vals = [float(r + 1) for r in range(15)] + [-1.0]
    ell_cols = list(range(15)) + [0]
    coo_vals = [-float(c + 1) for c in range(1, 16)]
    coo_rc = bytes([(15 << 4) | c for c in range(1, 16)])
    nib = bytes([ell_cols[2 * j] | (ell_cols[2 * j + 1] << 4) for j in range(8)])
    assert T.payload.tobytes() == pad16(f64(*ell_vals) + f64(*coo_vals) + nib + coo_rc)
    # DeferredCOO: the COO part moves to the remainder, the rest is ELL(1)
    Td = O.tile(A, "DEFERRED")
    assert (Td.tileFmt[0], Td.tileAux[0], Td.tileNnz[1]) == (ELL, 1, 16)
    assert Td.payload.tobytes() == pad16(f64(*ell_vals) + nib)
    assert Td.rem_nnz == 15 and list(Td.remCol) == list(range(1, 16))


def test_dns_payload_column_major():
    ents = [(r, c, r + c / 16.0 + 1.0) for r in range(16) for c in range(16) if (r + c) % 2 == 0 or r < 4]
    T = O.tile(one_tile(ents), "ADPT")
    assert T.tileFmt[0] == DNS
    vals = [0.0] * 256
    for r, c, v in ents:
        vals[16 * c + r] = v   # column-major
    assert T.payload.tobytes() == f64(*vals)


def test_dnsrow_third_row():
    # Fig. 3: the DnsRow tile's entries are all in the third row; its row id
    # is recorded (fragment "dnsrowldx 2" P:85) -> 0-based id 2
    T = O.tile(one_tile([(2, c, c + 0.5) for c in range(16)]), "ADPT")
    assert (T.tileFmt[0], T.tileAux[0]) == (DNSROW, 1)
    assert T.payload.tobytes() == pad16(f64(*[c + 0.5 for c in range(16)]) + bytes([2]))


def test_dnscol_two_columns():
    ents = [(r, c, 10.0 * c + r) for r in range(16) for c in (4, 11)]
    T = O.tile(one_tile(ents), "ADPT")
    assert (T.tileFmt[0], T.tileAux[0]) == (DNSCOL, 2)
    vals = [10.0 * 4 + r for r in range(16)] + [10.0 * 11 + r for r in range(16)]
    assert T.payload.tobytes() == pad16(f64(*vals) + bytes([4, 11]))


# --------------------------------------------------------------------------
# closed-form structure of the configs
# --------------------------------------------------------------------------

def test_lap2d_64_counts():
    """5-point Laplacian on 64x64: each 64-point x-line spans 4 tiles.
    Diagonal tiles (tridiagonal, lens {2,3x14,2}) -> ELL w=3: 256.
    J = I +- 4 (the +-64 couplings, identity blocks) -> ELL w=1: 2*(256-4).
    J = I +- 1 inside a line (one corner entry) -> COO: 64 lines * 3 * 2."""
    A, _ = gen.make("lap2d_64")
    T = O.tile(A, "ADPT")
    assert T.numtile == 256 + 504 + 384
    assert list(T.sel_tiles) == [0, 384, 760, 0, 0, 0, 0]
    w = T.tileAux[T.tileFmt == ELL]
    assert (w == 3).sum() == 256 and (w == 1).sum() == 504
    # payload: ELL w=3 -> 408 -> 416 B; ELL w=1 -> 136 -> 144 B; COO 1 nnz -> 16 B
    assert T.payload_bytes == 256 * 416 + 504 * 144 + 384 * 16 == 185216
    Td = O.tile(A, "DEFERRED")
    assert Td.numtile == 760 and Td.rem_nnz == 384
    assert Td.payload_bytes == 256 * 416 + 504 * 144


def test_fem_counts():
    """Tiles |J - I| <= 2: 5 per tile row minus the 6 that fall off the ends;
    dense tiles have 256 entries, the two triangles 136 each -> all Dns."""
    T_rows = 3904
    A, _ = gen.make("fem")
    T = O.tile(A, "DEFERRED")
    assert T.numtile == 5 * T_rows - 6 == 19514
    assert T.kept_tiles[DNS] == 19514 and T.rem_nnz == 0
    nnz = T_rows * (3 * 256 + 2 * 136) - 2 * (256 + 136) - 2 * 136
    assert A.nnz == nnz == 4059104
    assert T.payload_bytes == 19514 * 2048


def test_stencil27_48_counts():
    """48 = 0 mod 16: every x-line of 48 points spans 3 whole tiles.  For each
    line (y, z) and each in-range (dy, dz) neighbour plane: 3 tridiagonal
    tiles (ELL w=3) and 4 single-corner tiles (COO).  In-range (line, plane)
    pairs: (3*48 - 2)^2 = 142^2."""
    A, _ = gen.make("stencil27_48")
    assert A.nnz == 142 ** 3
    T = O.tile(A, "ADPT")
    pairs = 142 * 142
    assert list(T.sel_tiles) == [0, 4 * pairs, 3 * pairs, 0, 0, 0, 0]
    assert (T.tileAux[T.tileFmt == ELL] == 3).all()


def test_mixed_small_counts():
    """Per tile row: Dns, DnsRow(4), DnsCol(4), ELL(7), CSR, HYB(1), 10 COO."""
    A, _ = gen.make("mixed_small")
    T = O.tile(A, "ADPT")
    R = 64
    assert list(T.sel_tiles) == [R, 10 * R, R, R, R, R, R]
    assert T.sel_nnz[DNS] == 256 * R and T.sel_nnz[DNSROW] == 64 * R
    assert T.sel_nnz[DNSCOL] == 64 * R and T.sel_nnz[ELL] == 112 * R
    assert T.sel_nnz[CSR] == 96 * R and T.sel_nnz[HYB] == 44 * R
    assert set(T.tileAux[T.tileFmt == DNSROW]) == {4}
    assert set(T.tileAux[T.tileFmt == HYB]) == {1}
    Td = O.tile(A, "DEFERRED")
    # HYB w=1 -> ELL(1) (16 entries) + 28 extracted; all COO extracted
    assert Td.kept_tiles[ELL] == 2 * R and Td.kept_tiles[HYB] == 0
    assert Td.rem_nnz == T.sel_nnz[COO] + 28 * R


# --------------------------------------------------------------------------
# invariants + decode round trip
# --------------------------------------------------------------------------

def _size(fmt, aux, held):
    return {CSR: 8 * held + 16 + (held + 1) // 2, COO: 9 * held, ELL: 136 * aux,
            HYB: 136 * aux + 9 * (held - 16 * aux), DNS: 2048,
            DNSROW: 129 * aux, DNSCOL: 129 * aux}[fmt]


def check_invariants(A, T):
    assert T.tilem == (A.m + 15) // 16
    assert T.tilePtr[0] == 0 and T.tilePtr[-1] == T.numtile
    assert np.all(np.diff(T.tilePtr) >= 0)
    for I in range(T.tilem):
        cj = T.tileColIdx[T.tilePtr[I]:T.tilePtr[I + 1]]
        assert np.all(np.diff(cj) > 0)
    held = np.diff(T.tileNnz.astype(np.int64))
    assert np.all(held > 0)
    assert held.sum() + T.rem_nnz == A.nnz
    sizes = np.diff(T.tileOff.astype(np.int64)) * 16
    for t in range(T.numtile):
        s = _size(int(T.tileFmt[t]), int(T.tileAux[t]), int(held[t]))
        assert sizes[t] == (s + 15) // 16 * 16
        if T.tileFmt[t] in (ELL, HYB):
            assert 0 <= T.tileAux[t] <= 16
        if T.tileFmt[t] in (DNSROW, DNSCOL):  # paper rules: <= 7 (8 full rows = 128 -> Dns)
            assert 1 <= T.tileAux[t] <= (15 if T.mode == O.MODES["BYTES"] else 7)
    assert T.payload_bytes == T.tileOff[-1] * 16
    assert T.remRowPtr[-1] == T.rem_nnz


MATS = [
    ("lap2d_64", None), ("lap2d_37x29", None), ("fem_small", None), ("rmat12", None),
    ("mixed_small", None), ("stencil27_21", None),
]


def _special():
    yield gen.random_sparse(17, 33, 0.3, seed=1)
    yield gen.random_sparse(100, 1, 0.5, seed=2)
    yield gen.random_sparse(1, 100, 0.5, seed=3)
    yield gen.random_sparse(70, 70, 0.95, seed=4, empty_rows=range(16, 32))
    yield gen.random_sparse(130, 90, 0.05, seed=5)
    yield gen.dense(48, 40, seed=6)
    yield gen.random_sparse(0, 10, 0.5)
    yield gen.random_sparse(10, 0, 0.5)
    yield gen.random_sparse(33, 47, 0.0)


def _all_mats():
    for name, _ in MATS:
        yield gen.make(name)[0]
    yield from _special()


@pytest.mark.parametrize("mode", ["ADPT", "DEFERRED", "FORCE_CSR", "AUTO", "BYTES"])
def test_roundtrip_and_invariants(mode):
    for A in _all_mats():
        T = O.tile(A, mode)
        check_invariants(A, T)
        r, c, v = O.decode(A, mode)
        rows = np.repeat(np.arange(A.m), np.diff(A.rowptr))
        assert np.array_equal(r, rows), A.name
        assert np.array_equal(c, A.colidx), A.name
        assert np.array_equal(v.view(np.uint64), A.val.view(np.uint64)), A.name
        if mode == "FORCE_CSR":
            assert set(np.unique(T.tileFmt)) <= {CSR} and T.rem_nnz == 0
        if mode in ("ADPT", "BYTES"):
            assert T.rem_nnz == 0


def test_remainder_is_exactly_the_coo_data():
    """DEFERRED extracts every COO tile and the COO part of every HYB tile
    (P:201), and nothing else."""
    for A in _all_mats():
        Ta = O.tile(A, "ADPT")
        Td = O.tile(A, "DEFERRED")
        fmt_of = {}
        for I in range(Ta.tilem):
            for t in range(Ta.tilePtr[I], Ta.tilePtr[I + 1]):
                fmt_of[(I, int(Ta.tileColIdx[t]))] = (int(Ta.tileFmt[t]), int(Ta.tileAux[t]))
        expect = set()
        for i in range(A.m):
            cols = A.colidx[A.rowptr[i]:A.rowptr[i + 1]]
            rank = {}
            for c in cols:
                key = (i // 16, int(c) // 16)
                f, w = fmt_of[key]
                k = rank.get(key, 0)
                rank[key] = k + 1
                if f == COO or (f == HYB and k >= w):
                    expect.add((i, int(c)))
        got = set()
        for i in range(A.m):
            for k in range(Td.remRowPtr[i], Td.remRowPtr[i + 1]):
                got.add((i, int(Td.remCol[k])))
        assert got == expect, A.name


def test_explicit_zeros():
    """Explicit zeros are entries (R2, R27): counted for selection; a +0.0
    inside a Dns tile is indistinguishable from fill after decoding."""
    ents = [(r, c, 1.0 + r) for r in range(16) for c in range(16) if c < 9]
    ents[5] = (ents[5][0], ents[5][1], 0.0)
    ents[6] = (ents[6][0], ents[6][1], -0.0)
    A = one_tile(ents)
    T = O.tile(A, "ADPT")
    assert T.tileFmt[0] == DNS and T.tileNnz[1] == 144
    r, c, v = O.decode(A, "ADPT")
    assert len(r) == 143   # the +0.0 entry vanished, -0.0 survived (bit copy)
    assert np.signbit(v[(r == ents[6][0]) & (c == ents[6][1])]).all()
    # a COO tile keeps its explicit zero
    A2 = one_tile([(1, 1, 0.0), (2, 3, 5.0)])
    r2, c2, v2 = O.decode(A2, "ADPT")
    assert len(r2) == 2


def test_noncanonical_rejected():
    A = gen.random_sparse(20, 20, 0.5, seed=3)
    bad = gen.CSR(A.m, A.n, A.rowptr.copy(), A.colidx.copy(), A.val.copy())
    k = A.rowptr[2]
    bad.colidx[k], bad.colidx[k + 1] = bad.colidx[k + 1], bad.colidx[k]
    with pytest.raises(ValueError):
        O.tile(bad)
    bad2 = gen.CSR(A.m, A.n, A.rowptr.copy(), A.colidx.copy(), A.val.copy())
    bad2.colidx[-1] = A.n
    with pytest.raises(ValueError):
        O.tile(bad2)


def test_auto_switch_at_1_8M():
    """AUTO: DeferredCOO above the 1.8M size of P:235 (reading R18: nnz)."""
    A, _ = gen.make("stencil27_40")      # 1,643,032 nnz
    assert O.tile(A, "AUTO").mode == 0
    B, _ = gen.make("stencil27_48")      # 2,863,288 nnz
    assert O.tile(B, "AUTO").mode == 1


def test_golden_counts_match_oracle():
    """tests/golden/config_counts.json was written by
    tests/golden/make_golden.py, which calls only oracle/.  Re-check the
    small entries here (the large ones are re-checked on the GPU box)."""
    with open(os.path.join(GOLDEN, "config_counts.json")) as f:
        gold = json.load(f)
    for name in ("lap2d_64", "fem_small", "rmat12", "mixed_small", "stencil27_40"):
        A, _ = gen.make(name)
        for mode in ("ADPT", "DEFERRED"):
            T = O.tile(A, mode)
            g = gold[name][mode]
            assert g["numtile"] == T.numtile
            assert g["sel_tiles"] == T.sel_tiles.tolist()
            assert g["kept_tiles"] == T.kept_tiles.tolist()
            assert g["payload_bytes"] == T.payload_bytes
            assert g["rem_nnz"] == T.rem_nnz
            assert g["nnz"] == A.nnz


# --------------------------------------------------------------------------
# optional B200 byte-cost selection (not the paper's rule):
# hand-computed payload sizes (rounded to 16) at its boundaries
# --------------------------------------------------------------------------

def _masks_full_rows(full, extra=()):
    m = [0xFFFF if r in full else 0 for r in range(16)]
    for r, cols in extra:
        for c in cols:
            m[r] |= 1 << c
    return m


@pytest.mark.parametrize("masks,fmt,aux,why", [
    # FEM's upper-triangle tile (row r holds columns r..15, 136 entries): CSR
    # 8*136+16+68 = 1172 -> 1184 beats Dns 2048, ELL 16*136 = 2176, HYB(w=1)
    # 136+9*120 = 1216, COO 1224 (the paper's rule takes Dns: n >= 128)
    ([(0xFFFF << r) & 0xFFFF for r in range(16)], CSR, 0, "triangle"),
    # a full tile: Dns 2048 < DnsRow/DnsCol 2064 < CSR 2192
    ([0xFFFF] * 16, DNS, 0, "full"),
    # 13 full rows + rows of 15, 15 and 1 = 239 entries: CSR 1912+16+120 =
    # 2048 ties Dns 2048 and the lower code wins (HYB w=1: 2143 -> 2144)
    (_masks_full_rows(range(13), [(13, range(15)), (14, range(1, 16)), (15, [0])]), CSR, 0, "239"),
    # ... and 240 (last row of 2): CSR 1920+16+120 = 2056 -> 2064 > Dns 2048
    (_masks_full_rows(range(13), [(13, range(15)), (14, range(1, 16)), (15, [0, 1])]), DNS, 0, "240"),
    # one entry: COO 9 -> 16 beats CSR 25 -> 32
    ([1] + [0] * 15, COO, 0, "single"),
    # one full row: COO 144 ties DnsRow 129 -> 144; the lower code (COO) wins
    (_masks_full_rows([5]), COO, 0, "one full row"),
    # 3 full rows: DnsRow 387 -> 400 beats COO 432, CSR 384+16+24 = 424 -> 432
    (_masks_full_rows([1, 7, 12]), DNSROW, 3, "three full rows"),
    # 16 rows of 3: ELL 408 -> 416 ties HYB(w=3) 408 -> 416 and beats CSR
    # 424 -> 432 and COO 432: ELL (lower code)
    ([0b111 << (r % 14) for r in range(16)], ELL, 3, "equal rows of 3"),
    # 15 rows of 3 and an empty row: ELL not eligible (R26), HYB w=0 = COO
    # 405 -> 416, CSR 360+16+23 = 399 -> 400
    ([0b111 << (r % 14) for r in range(15)] + [0], CSR, 0, "empty row"),
])
def test_select_bytes_boundaries(masks, fmt, aux, why):
    assert O.select_bytes(masks) == (fmt, aux), why


def test_select_bytes_is_a_minimum_over_brute_force_layouts():
    """On random tiles, the byte rule's choice has the smallest payload of the
    formats that can hold the tile, sizes taken from the oracle's own packing
    of single-tile matrices in each format (BYTES, ADPT, FORCE_CSR tilings)."""
    rng = np.random.default_rng(5)
    for trial in range(300):
        dens = rng.choice([0.02, 0.1, 0.3, 0.6, 0.95])
        M = (rng.random((16, 16)) < dens)
        if not M.any():
            continue
        masks = [int(sum(1 << c for c in range(16) if M[r, c])) for r in range(16)]
        f, a = O.select_bytes(masks)
        A = gen.from_dense(np.where(M, 1.0 + rng.random((16, 16)), 0.0))
        Tb = O.tile(A, "BYTES")
        assert Tb.numtile == 1 and int(Tb.tileFmt[0]) == f and int(Tb.tileAux[0]) == a
        got = int(Tb.payload_bytes)
        # the paper's choice and plain CSR are never smaller
        for mode in ("ADPT", "FORCE_CSR"):
            assert got <= int(O.tile(A, mode).payload_bytes), (trial, mode)
