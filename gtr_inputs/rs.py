"""RSBench-style windowed multipole tables (config 4).

Recipe (the paper names the app and its
command line only; structure per RSBench [ext]):

* n_nuc nuclides (355), avg_poles = 1000, avg_windows = 100, numL = 4.
* n_poles[n]: every nuclide gets 1, the remaining avg*n_nuc - n_nuc poles go to
  nuclide floor(U * n_nuc) each (multinomial); same for n_windows.
* poles (padded to max_poles per nuclide): EA, RT, RA, RF complex, each part
  U; l_value = floor(U * numL).
* windows: T, A, F = U; pole ranges split n_poles as evenly as possible, the
  first (n_poles mod n_windows) windows one pole longer; `end` is stored as in
  RSBench (last pole index, inclusive) -- the method loops i in [start, end).
* pseudo_K0RS[n][4] = U.
* Materials and concentrations as XS large (355 nuclides).

All draws come from one table stream (SEED_RS) consumed block by block in the
order above.
"""
import numpy as np

from .stream import uniform
from .xs import material_lists, N_MATS

SEED_RS = 42
SEED_C = 13
NUM_L = 4

POLE_DTYPE = np.dtype([("EA", "<f8", 2), ("RT", "<f8", 2), ("RA", "<f8", 2),
                       ("RF", "<f8", 2), ("l_value", "<i4"), ("pad", "<i4")])   # 72 B
WIN_DTYPE = np.dtype([("T", "<f8"), ("A", "<f8"), ("F", "<f8"),
                      ("start", "<i4"), ("end", "<i4")])                         # 32 B


def _multinomial(seed, n_nuc, avg):
    u = uniform(seed, avg * n_nuc - n_nuc)
    idx = (u * n_nuc).astype(np.int64)
    return (np.bincount(idx, minlength=n_nuc) + 1).astype(np.int32)


def make_tables(n_nuc=355, avg_poles=1000, avg_windows=100, seed=SEED_RS,
                seed_c=SEED_C):
    n_poles = _multinomial(seed, n_nuc, avg_poles)
    n_windows = _multinomial(seed + 1, n_nuc, avg_windows)
    max_poles = int(n_poles.max())
    max_windows = int(n_windows.max())

    tot_p = int(n_poles.sum())
    u = uniform(seed + 2, tot_p * 9)
    poles = np.zeros((n_nuc, max_poles), dtype=POLE_DTYPE)
    k = 0
    for n in range(n_nuc):
        c = int(n_poles[n])
        blk = u[k * 9:(k + c) * 9].reshape(c, 9)
        poles["EA"][n, :c] = blk[:, 0:2]
        poles["RT"][n, :c] = blk[:, 2:4]
        poles["RA"][n, :c] = blk[:, 4:6]
        poles["RF"][n, :c] = blk[:, 6:8]
        poles["l_value"][n, :c] = (blk[:, 8] * NUM_L).astype(np.int32)
        k += c

    tot_w = int(n_windows.sum())
    u = uniform(seed + 3, tot_w * 3)
    windows = np.zeros((n_nuc, max_windows), dtype=WIN_DTYPE)
    k = 0
    for n in range(n_nuc):
        nw = int(n_windows[n])
        space = int(n_poles[n]) // nw
        rem = int(n_poles[n]) - space * nw
        ctr = 0
        for j in range(nw):
            windows["T"][n, j] = u[(k + j) * 3 + 0]
            windows["A"][n, j] = u[(k + j) * 3 + 1]
            windows["F"][n, j] = u[(k + j) * 3 + 2]
            start = ctr
            end = ctr + space - 1
            ctr += space
            if j < rem:
                ctr += 1
                end += 1
            windows["start"][n, j] = start
            windows["end"][n, j] = end
        k += nw

    k0rs = uniform(seed + 4, n_nuc * NUM_L).reshape(n_nuc, NUM_L)

    lists = material_lists(355 if n_nuc == 355 else n_nuc)
    num_nucs = np.array([len(l) for l in lists], dtype=np.int32)
    max_nn = int(num_nucs.max())
    mats = np.full((N_MATS, max_nn), -1, dtype=np.int32)
    concs = np.zeros((N_MATS, max_nn), dtype=np.float64)
    cdraw = uniform(seed_c, int(num_nucs.sum()))
    k = 0
    for m, l in enumerate(lists):
        mats[m, :len(l)] = l
        concs[m, :len(l)] = cdraw[k:k + len(l)]
        k += len(l)
    return {"n_nuc": n_nuc, "n_poles": n_poles, "n_windows": n_windows,
            "poles": poles, "windows": windows, "k0rs": k0rs,
            "num_nucs": num_nucs, "mats": mats, "concs": concs,
            "max_poles": max_poles, "max_windows": max_windows}
