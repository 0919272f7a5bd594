"""Writes tests/golden/config_counts.json: tile/format counts of the synthetic
configs under the reference tiler.  Calls ONLY oracle/ (and the shared input
generators), never the CUDA path, so the stored values are oracle values.

    python tests/golden/make_golden.py              # small configs
    python tests/golden/make_golden.py --large      # + the full BASELINE configs
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

from oracle import oracle as O  # noqa: E402
from synthetic import gen  # noqa: E402

SMALL = ["lap2d_64", "lap2d_37x29", "fem_small", "rmat12", "mixed_small",
         "stencil27_21", "stencil27_40", "stencil27_48"]
LARGE = ["fem", "rmat20", "mixed", "stencil27_200"]


def counts(name):
    A, _ = gen.make(name)
    out = {}
    for mode in ("ADPT", "DEFERRED"):
        T = O.tile(A, mode)
        out[mode] = dict(nnz=A.nnz, numtile=T.numtile, sel_tiles=T.sel_tiles.tolist(),
                         sel_nnz=T.sel_nnz.tolist(), kept_tiles=T.kept_tiles.tolist(),
                         kept_nnz=T.kept_nnz.tolist(), payload_bytes=T.payload_bytes,
                         rem_nnz=T.rem_nnz)
        del T
    return out


def main():
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "config_counts.json")
    gold = {}
    if os.path.exists(path):
        with open(path) as f:
            gold = json.load(f)
    names = SMALL + (LARGE if "--large" in sys.argv else [])
    for name in names:
        gold[name] = counts(name)
        print(name, gold[name]["DEFERRED"]["numtile"], flush=True)
        with open(path, "w") as f:
            json.dump(gold, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
