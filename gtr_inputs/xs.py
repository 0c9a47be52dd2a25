"""XSBench-style continuous-energy cross-section tables (configs 1 and 5).

Recipe (the paper only names the app and its
command line):

* n_iso nuclides (68 "small", 355 "large") x n_gp = 11,303 gridpoints each.
* For every point, in order, six uniform draws from the table stream seeded
  with SEED_T = 42: energy, total, elastic, absorption, fission, nu_fission.
* Each nuclide's points are sorted by (energy, original index) -- a nuclide's
  cross-section table is ordered by energy.
* 12 materials with num_nucs = {34|321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9}
  and XSBench's hard-coded nuclide lists ([ext], recalled, unverified); the
  large fuel list appends nuclides 68..354.
* Concentrations: uniform draws in (material, slot) order from SEED_C = 13.

Returned arrays are C-contiguous numpy arrays.  The unionized energy grid and
the index grid are NOT built here: they are part of the method (the
"unionized grid" acceleration structure) and each side builds its own.
"""
import numpy as np

from .stream import uniform

N_GRIDPOINTS = 11303
SEED_T = 42
SEED_C = 13
SEED_L = 1070          # lookup stream seed (consumed by the method, not here)
N_MATS = 12

_FUEL_SMALL = [58, 59, 60, 61, 40, 42, 43, 44, 45, 46, 1, 2, 3, 7, 8, 9, 10,
               29, 57, 47, 48, 0, 62, 15, 33, 34, 52, 53, 54, 55, 56, 18, 23, 41]
_CLAD = [63, 64, 65, 66, 67]
_WATER = [24, 41, 4, 5]
_RPV = [19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30, 31, 32, 26,
        49, 50, 51, 11, 12, 13, 14, 6, 16, 17]
_REFL = [24, 41, 4, 5, 19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30,
         31, 32, 26]
_PLENUM = [24, 41, 4, 5, 63, 64, 65, 66, 67]


def material_lists(n_iso):
    """The 12 nuclide lists (python lists of ints)."""
    if n_iso == 68:
        fuel = list(_FUEL_SMALL)
    elif n_iso == 355:
        fuel = list(_FUEL_SMALL) + list(range(68, 355))
    else:
        # generic sizes (tests): fuel = every nuclide, others clipped to range
        fuel = list(range(n_iso))
    lists = [fuel, _CLAD, _WATER, _WATER, _RPV, _REFL, _REFL, _REFL, _REFL,
             _REFL, _PLENUM, _PLENUM]
    if n_iso not in (68, 355):
        lists = [fuel] + [[n % n_iso for n in l] for l in lists[1:]]
        lists = [list(dict.fromkeys(l)) for l in lists]   # drop duplicates
    return lists


def make_tables(n_iso, n_gp=N_GRIDPOINTS, seed_t=SEED_T, seed_c=SEED_C):
    """Generate one XS problem.  Returns a dict of numpy arrays:

    grid      f64 [n_iso, n_gp, 6]  (energy, total, elastic, absorption,
                                     fission, nu_fission), each nuclide sorted
    num_nucs  i32 [12]
    mats      i32 [12, max_num_nucs] (row m valid up to num_nucs[m]; rest -1)
    concs     f64 [12, max_num_nucs] (rest 0)
    """
    raw = uniform(seed_t, n_iso * n_gp * 6).reshape(n_iso, n_gp, 6)
    order = np.argsort(raw[:, :, 0], axis=1, kind="stable")
    grid = np.take_along_axis(raw, order[:, :, None], axis=1)
    grid = np.ascontiguousarray(grid)

    lists = material_lists(n_iso)
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
    return {"grid": grid, "num_nucs": num_nucs, "mats": mats, "concs": concs,
            "n_iso": n_iso, "n_gp": n_gp}


def constructed_tables(n_iso, n_gp, dominant, seed=7):
    """Tables where channel `dominant` exceeds all others at every point
    (used by the hash pins): values of that channel are drawn
    in [10, 11), the others in [0, 1)."""
    t = make_tables(n_iso, n_gp, seed_t=seed, seed_c=seed + 1)
    g = t["grid"]
    g[:, :, 1 + dominant] += 10.0
    return t
