"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module is the ONE piece of code both sides may use.  It builds problem data
(random arrays, proxy-app lookup tables) and holds none of the method's arithmetic:
no schedule, no reduction, no lookup, no interpolation, no Faddeeva evaluation.
Everything the method itself draws at run time (the per-lookup LCG stream of
XSBench/RSBench) is implemented separately by `oracle/` and by the CUDA kernels.

Recipes:
  * splitmix64 streams for C1 (axpy), C2 (generic), C5 (SU(3)).
  * The XSBench/RSBench 63-bit LCG (m = 2^63, a = 2806196910506780709, c = 1)
    for the proxy-app tables, evaluated in closed form s_k = a^k s_0 + sum_{j<k} a^j
    (mod 2^63) with numpy uint64 wrap-around, which equals k sequential steps.

All functions are deterministic in their seed and return numpy arrays (host memory).
"""
from __future__ import annotations

import numpy as np

# --------------------------------------------------------------------------------------
# splitmix64 (Steele, Lea, Flood 2014) -- counter based, vectorised
# --------------------------------------------------------------------------------------
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """u64 outputs z_{offset+1} .. z_{offset+n} of splitmix64 seeded with `seed`."""
    with np.errstate(over="ignore"):
        k = np.arange(offset + 1, offset + n + 1, dtype=np.uint64)
        z = np.uint64(seed) + k * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def u01(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """Doubles in [0,1): (splitmix64 >> 11) * 2^-53 (exact conversion)."""
    return (splitmix64(seed, n, offset) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def uniform(seed: int, n: int, lo: float, hi: float, offset: int = 0) -> np.ndarray:
    """Doubles in [lo,hi) as lo + (hi-lo)*u01 (exact when hi-lo is a power of two)."""
    return lo + (hi - lo) * u01(seed, n, offset)


# --------------------------------------------------------------------------------------
# C1: SPMD axpy + sum inputs
# --------------------------------------------------------------------------------------
SEED_B = 0xB0B0B0B0
SEED_C = 0xC0C0C0C0


def axpy_inputs(n: int, exact: bool = False):
    """Returns (x, b, c).  exact=True: x=2, b[i]=i mod 1024, c[i]=1 (integer valued)."""
    if exact:
        b = (np.arange(n, dtype=np.int64) % 1024).astype(np.float64)
        return 2.0, b, np.ones(n, dtype=np.float64)
    return 1.5, u01(SEED_B, n), u01(SEED_C, n)


# --------------------------------------------------------------------------------------
# C2: generic-mode synthetic inputs
# --------------------------------------------------------------------------------------
SEED_GENERIC = 0x6E6E6E6E


def generic_inputs(teams: int, inner_n: int) -> np.ndarray:
    return u01(SEED_GENERIC, teams * inner_n)


# --------------------------------------------------------------------------------------
# C5: SU(3) inputs.  Layout: site-major AoS
#     A[site][link 0..3][row 0..2][col 0..2][re,im]  (72 doubles = 576 B per site)
#     B[link][row][col][re,im]                        (72 doubles)
# --------------------------------------------------------------------------------------
SEED_SU3_A = 0x5A5A5A5A
SEED_SU3_B = 0x5B5B5B5B
SU3_DOUBLES_PER_SITE = 4 * 3 * 3 * 2


def su3_inputs(n_sites: int, kind: str = "random", first_site: int = 0):
    """kind: 'random' (U[-1,1)), 'identity' (B = I), 'third' (A = 1+0i, B = 1/3+0i).
    first_site: A for sites [first_site, first_site + n_sites) of the same lattice (a
    rank's contiguous shard)."""
    if kind == "random":
        a = uniform(SEED_SU3_A, n_sites * SU3_DOUBLES_PER_SITE, -1.0, 1.0,
                    first_site * SU3_DOUBLES_PER_SITE)
        b = uniform(SEED_SU3_B, SU3_DOUBLES_PER_SITE, -1.0, 1.0)
    elif kind == "identity":
        a = uniform(SEED_SU3_A, n_sites * SU3_DOUBLES_PER_SITE, -1.0, 1.0)
        b = np.zeros((4, 3, 3, 2))
        for l in range(4):
            for r in range(3):
                b[l, r, r, 0] = 1.0
        b = b.reshape(-1)
    elif kind == "third":
        a = np.zeros((n_sites, 4, 3, 3, 2))
        a[..., 0] = 1.0
        a = a.reshape(-1)
        b = np.zeros((4, 3, 3, 2))
        b[..., 0] = 1.0 / 3.0
        b = b.reshape(-1)
    else:
        raise ValueError(kind)
    return np.ascontiguousarray(a), np.ascontiguousarray(b)


# --------------------------------------------------------------------------------------
# The proxy apps' 63-bit LCG, used here only to build TABLES (problem data)
# --------------------------------------------------------------------------------------
LCG_A = 2806196910506780709
LCG_C = 1
_MASK63 = np.uint64((1 << 63) - 1)


def lcg_states(seed: int, n: int) -> np.ndarray:
    """States s_1..s_n of s_{k+1} = (a s_k + 1) mod 2^63 from s_0 = seed (uint64 array).

    Closed form s_k = a^k s_0 + (1 + a + ... + a^{k-1}) mod 2^63; cumprod/cumsum wrap mod
    2^64 and 2^63 divides 2^64, so masking the low 63 bits gives the mod-2^63 value.
    """
    if n == 0:
        return np.zeros(0, dtype=np.uint64)
    with np.errstate(over="ignore"):
        pw = np.cumprod(np.full(n, LCG_A, dtype=np.uint64))          # a^1 .. a^n
        geo = np.empty(n, dtype=np.uint64)                            # sum_{j<k} a^j, k=1..n
        geo[0] = 1
        if n > 1:
            geo[1:] = np.uint64(1) + np.cumsum(pw[:-1])
        s = pw * np.uint64(seed) + geo * np.uint64(LCG_C)
        return s & _MASK63


def lcg_doubles(seed: int, n: int):
    """(doubles, final_state): LCG_random_double drawn n times = (double)s / 2^63."""
    s = lcg_states(seed, n)
    d = s.astype(np.float64) * (2.0 ** -63)
    return d, (int(s[-1]) if n else seed)


# --------------------------------------------------------------------------------------
# Materials shared by XSBench and RSBench (XSBench's fixed lists [ext])
# --------------------------------------------------------------------------------------
FUEL_SMALL = [58, 59, 60, 61, 40, 42, 43, 44, 45, 46, 1, 2, 3, 7, 8, 9, 10, 29, 57, 47, 48, 0,
              62, 15, 33, 34, 52, 53, 54, 55, 56, 18, 23, 41]
CLADDING = [63, 64, 65, 66, 67]
WATER = [24, 41, 4, 5]
RPV = [19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30, 31, 32, 26, 49, 50, 51, 11, 12, 13,
       14, 6, 16, 17]
MAT_5_9 = [24, 41, 4, 5, 19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 49, 50, 51, 11, 12, 13, 14]
MAT_10_11 = [24, 41, 4, 5, 63, 64, 65, 66, 67]
# pick_mat's distribution (XSBench/RSBench), listed by material id
MAT_DIST = [0.140, 0.052, 0.275, 0.134, 0.154, 0.064, 0.066, 0.055, 0.008, 0.015, 0.025, 0.013]


def material_lists(large: bool):
    fuel = FUEL_SMALL + (list(range(68, 355)) if large else [])
    return [fuel, CLADDING, WATER, WATER, RPV] + [MAT_5_9] * 5 + [MAT_10_11] * 2


def materials(large: bool, concs_seed: int):
    """(num_nucs int32[12], mats int32[12*max], concs f64[12*max], max_num_nucs).

    concs: LCG doubles drawn in (material, nuclide) order from `concs_seed`."""
    lists = material_lists(large)
    mx = max(len(l) for l in lists)
    num = np.array([len(l) for l in lists], dtype=np.int32)
    mats = np.zeros((12, mx), dtype=np.int32)
    for m, l in enumerate(lists):
        mats[m, : len(l)] = l
    total = int(num.sum())
    d, _ = lcg_doubles(concs_seed, total)
    concs = np.zeros((12, mx), dtype=np.float64)
    k = 0
    for m in range(12):
        concs[m, : num[m]] = d[k: k + num[m]]
        k += num[m]
    return num, mats.reshape(-1), concs.reshape(-1), mx


# --------------------------------------------------------------------------------------
# C3: XSBench-shaped tables
# --------------------------------------------------------------------------------------
XS_GRID_SEED = 42
XS_CONCS_SEED = 0xC0C5
XS_LOOKUP_SEED = 1070  # STARTING_SEED: consumed by the method (oracle / kernels), not here
XS_SMALL = dict(n_isotopes=68, n_gridpoints=11303, large=False)


class XSTables:
    """XSBench unionized-grid tables.

    nuclide_grid : f64 [n_isotopes*n_gridpoints, 6]  (energy, total, elastic, absorption,
                   fission, nu_fission), each nuclide's block sorted by energy
    unionized    : f64 [n_isotopes*n_gridpoints]     all energies, sorted
    index_grid   : i32 [len(unionized), n_isotopes]  per unionized energy, per nuclide, the
                   lower bracket index into that nuclide's block (clamped to [0, n_gp-2])
    num_nucs/mats/concs : materials (see `materials`)
    """

    def __init__(self, n_isotopes=68, n_gridpoints=11303, large=False, seed=XS_GRID_SEED,
                 concs_seed=XS_CONCS_SEED):
        self.n_isotopes, self.n_gridpoints = n_isotopes, n_gridpoints
        npts = n_isotopes * n_gridpoints
        d, _ = lcg_doubles(seed, 6 * npts)
        g = d.reshape(n_isotopes, n_gridpoints, 6)
        order = np.argsort(g[:, :, 0], axis=1, kind="stable")
        g = np.take_along_axis(g, order[:, :, None], axis=1)
        self.nuclide_grid = np.ascontiguousarray(g.reshape(npts, 6))
        self.unionized = np.sort(g[:, :, 0].reshape(-1), kind="stable")
        ig = np.empty((npts, n_isotopes), dtype=np.int32)
        for i in range(n_isotopes):
            c = np.searchsorted(g[i, :, 0], self.unionized, side="right") - 1
            ig[:, i] = np.clip(c, 0, n_gridpoints - 2)
        self.index_grid = ig
        (self.num_nucs, self.mats, self.concs, self.max_num_nucs) = materials(large, concs_seed)

    @property
    def n_union(self):
        return self.unionized.shape[0]

    @property
    def index_grid16(self):
        """The same index grid as uint16 (every entry is < n_gridpoints <= 65536): the
        compact host-side layout of the data (a copy, made on first use)."""
        if not hasattr(self, "_ig16"):
            assert self.n_gridpoints <= 65536
            self._ig16 = self.index_grid.astype(np.uint16)
        return self._ig16

    def nbytes(self):
        return (self.nuclide_grid.nbytes + self.unionized.nbytes + self.index_grid.nbytes
                + self.num_nucs.nbytes + self.mats.nbytes + self.concs.nbytes)


def xs_tied_channels(t: "XSTables") -> "XSTables":
    """A copy of XS tables with channels made equal at every gridpoint: elastic := total,
    fission := nu-fission := absorption (columns 2 := 1, 4 := 5 := 3).  Input data only:
    lookups on it accumulate equal macroscopic values, so ties in the argmax are certain."""
    import copy
    c = copy.copy(t)
    g = t.nuclide_grid.reshape(-1, 6).copy()
    g[:, 2] = g[:, 1]
    g[:, 4] = g[:, 3]
    g[:, 5] = g[:, 3]
    c.nuclide_grid = np.ascontiguousarray(g.reshape(t.nuclide_grid.shape))
    return c


# --------------------------------------------------------------------------------------
# C4: RSBench-shaped multipole tables, CSR layout
# --------------------------------------------------------------------------------------
RS_SEED = 42
RS_CONCS_SEED = 0xC0C5
RS_LOOKUP_SEED = 1070


class RSTables:
    """RSBench-shaped multipole tables (poles and windows in CSR order per nuclide).

    poles      : f64 [n_poles_total, 8]  EA.re EA.im RT.re RT.im RA.re RA.im RF.re RF.im
    pole_l     : i32 [n_poles_total]     l_value in [0, numL)
    windows    : f64 [n_windows_total, 4] T, A, F, 0
    win_range  : i32 [n_windows_total, 2] absolute [start, end) pole indices
    win_off    : i32 [n_nuclides+1]       CSR offsets of each nuclide's windows
    n_windows  : i32 [n_nuclides]
    k0rs       : f64 [n_nuclides, numL]   pseudo_K0RS
    num_nucs/mats/concs : materials (large lists)
    """

    def __init__(self, n_nuclides=355, avg_poles=1000, avg_windows=100, numL=4, seed=RS_SEED,
                 concs_seed=RS_CONCS_SEED, large=True):
        self.n_nuclides, self.numL = n_nuclides, numL
        s = seed
        # n_poles: all start at 1, extras go to nuclide floor(LCG*n) one at a time
        extra = n_nuclides * avg_poles - n_nuclides
        d, s = lcg_doubles(s, extra)
        n_poles = 1 + np.bincount(np.minimum((d * n_nuclides).astype(np.int64), n_nuclides - 1),
                                  minlength=n_nuclides)
        extra_w = n_nuclides * avg_windows - n_nuclides
        d, s = lcg_doubles(s, extra_w)
        n_win = 1 + np.bincount(np.minimum((d * n_nuclides).astype(np.int64), n_nuclides - 1),
                                minlength=n_nuclides)
        n_win = np.minimum(n_win, n_poles)  # every window keeps >= 1 pole
        total_p = int(n_poles.sum())
        d, s = lcg_doubles(s, 9 * total_p)
        d = d.reshape(total_p, 9)
        poles = np.empty((total_p, 8))
        # EA = 152.5 (r - i im): Im EA <= 0 puts Z = (E - EA)/2 in the upper half plane,
        # where the Faddeeva approximations are valid (reading R-A2)
        poles[:, 0] = 152.5 * d[:, 0]
        poles[:, 1] = -152.5 * d[:, 1]
        for k, col in ((1, 2), (2, 4), (3, 6)):
            poles[:, col] = 152.5 * d[:, 2 * k]
            poles[:, col + 1] = d[:, 2 * k + 1]
        self.poles = np.ascontiguousarray(poles)
        self.pole_l = np.minimum((d[:, 8] * numL).astype(np.int32), numL - 1)
        pole_off = np.zeros(n_nuclides + 1, dtype=np.int64)
        pole_off[1:] = np.cumsum(n_poles)
        total_w = int(n_win.sum())
        d, s = lcg_doubles(s, 3 * total_w)
        win = np.zeros((total_w, 4))
        win[:, :3] = d.reshape(total_w, 3)
        self.windows = win
        rng = np.empty((total_w, 2), dtype=np.int32)
        win_off = np.zeros(n_nuclides + 1, dtype=np.int32)
        win_off[1:] = np.cumsum(n_win)
        for i in range(n_nuclides):
            nw, npl = int(n_win[i]), int(n_poles[i])
            space, rem = divmod(npl, nw)
            sizes = np.full(nw, space, dtype=np.int64)
            sizes[:rem] += 1
            ends = pole_off[i] + np.cumsum(sizes)
            rng[win_off[i]: win_off[i + 1], 1] = ends
            rng[win_off[i]: win_off[i + 1], 0] = ends - sizes
        self.win_range = rng
        self.win_off = win_off
        self.n_windows = n_win.astype(np.int32)
        self.n_poles = n_poles.astype(np.int32)
        d, s = lcg_doubles(s, n_nuclides * numL)
        self.k0rs = d.reshape(n_nuclides, numL).copy()
        (self.num_nucs, self.mats, self.concs, self.max_num_nucs) = materials(large, concs_seed)

    def nbytes(self):
        return sum(a.nbytes for a in (self.poles, self.pole_l, self.windows, self.win_range,
                                      self.win_off, self.k0rs, self.num_nucs, self.mats,
                                      self.concs))
