"""Seeded synthetic XGC-shaped batched linear systems (inputs only).

This module is the ONE piece shared by the CUDA path's tests/bench and by the
CPU oracle: it produces the shared sparsity pattern, the per-system matrix
values and right-hand sides.  It contains none of the solver's arithmetic
(no SpMV, no dot product, no preconditioner, no Krylov step); it only draws
numbers and lays them out.

Why synthetic: the paper's matrices come from the XGC Fokker-Planck-Landau
collision operator, which is not public (Data
availability).  The paper fixes the *shape* of the workload and this module
reproduces it:

* 992 rows, one 9-point stencil shared by every system in the batch
  (Sec. IV-A, Fig. 4; Sec. II-A).
* non-symmetric values.
* ion and electron species in equal numbers, interleaved by global system
  index: even g = ion, odd g = electron (Sec. V).
* ions have eigenvalues clustered near 1, electrons a wider spread of real
  parts, both well-conditioned (Fig. 2).
* Picard warm-start sequence (Table III).

The recipe is SURVEY.md section 8(d) and is restated in DESIGN.md
("Input recipe").  Every random number is a pure function of
(seed, global system index g, row r, field) through a counter-based
splitmix64 hash, so any slice of a batch is generated identically no matter
how the batch is partitioned across ranks or chunks.
"""
from __future__ import annotations

import concurrent.futures as cf
import dataclasses
import math
import os

import numpy as np

DEFAULT_SEED = 20220530

# splitmix64 constants (Steele, Lea, Flood 2014); used here only as a hash.
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

# Random fields per (g, r).  Two uniforms per normal (Box-Muller).
F_DXX_A, F_DXX_B, F_DYY_A, F_DYY_B, F_DXY, F_B_A, F_B_B = range(7)
_NFIELDS = 8  # field slots reserved per row (power of two)

# Stencil neighbour order == ascending column order in lexicographic numbering
# r = j*nx + i (i fast).  (di, dj) per type.
STENCIL = ((-1, -1), (0, -1), (1, -1),
           (-1, 0), (0, 0), (1, 0),
           (-1, 1), (0, 1), (1, 1))
CENTER = 4

ION_K = 0.05
ELECTRON_K = 8.0


def _mix64(z):
    z = z.copy() if isinstance(z, np.ndarray) else np.uint64(z)
    z ^= z >> np.uint64(30)
    z *= _M1
    z ^= z >> np.uint64(27)
    z *= _M2
    z ^= z >> np.uint64(31)
    return z


def hash_u64(seed: int, g: np.ndarray, r: np.ndarray, field: int) -> np.ndarray:
    """Counter-based 64-bit hash of (seed, g, r, field); broadcasting."""
    with np.errstate(over="ignore"):
        s = _mix64(np.uint64(seed) + _GOLDEN)
        a = _mix64(np.asarray(g, dtype=np.uint64) ^ s)
        c = (np.asarray(r, dtype=np.uint64) << np.uint64(3)) | np.uint64(field)
        return _mix64(a + c * _GOLDEN)


def uniform01(seed, g, r, field) -> np.ndarray:
    """Uniform in the open interval (0, 1), 53-bit resolution."""
    h = hash_u64(seed, g, r, field)
    return ((h >> np.uint64(11)).astype(np.float64) + 0.5) * (2.0 ** -53)


def normal(seed, g, r, field_a, field_b) -> np.ndarray:
    """Standard normal by Box-Muller from two counter-based uniforms."""
    u1 = uniform01(seed, g, r, field_a)
    u2 = uniform01(seed, g, r, field_b)
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * math.pi * u2)


@dataclasses.dataclass(frozen=True)
class Pattern:
    """Shared CSR sparsity pattern of the 9-point stencil on an nx-by-ny grid.

    row_ptr/col_idx are int32, columns sorted ascending inside each row.
    ``ntype[e]`` is the stencil neighbour type (index into STENCIL) of entry e.
    """
    nx: int
    ny: int
    row_ptr: np.ndarray
    col_idx: np.ndarray
    row_of: np.ndarray
    ntype: np.ndarray

    @property
    def n(self) -> int:
        return self.nx * self.ny

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def max_row_nnz(self) -> int:
        return int(np.max(np.diff(self.row_ptr)))


def stencil_pattern(nx: int = 32, ny: int = 31) -> Pattern:
    """9-point stencil, in-grid neighbours only (real boundary shape).

    nx is the fast dimension: row r = j*nx + i (reading R13).
    """
    rp = [0]
    cols, rows, types = [], [], []
    for j in range(ny):
        for i in range(nx):
            r = j * nx + i
            for t, (di, dj) in enumerate(STENCIL):
                ii, jj = i + di, j + dj
                if 0 <= ii < nx and 0 <= jj < ny:
                    cols.append(jj * nx + ii)
                    rows.append(r)
                    types.append(t)
            rp.append(len(cols))
    return Pattern(nx, ny, np.asarray(rp, np.int32), np.asarray(cols, np.int32),
                   np.asarray(rows, np.int32), np.asarray(types, np.int8))


@dataclasses.dataclass(frozen=True)
class Species:
    """Coefficients of the synthetic Fokker-Planck-like operator."""
    k: float                # diffusion strength: ion 0.05, electron 8.0
    cross: float = 0.5      # mixed-derivative strength (dxy)
    jitter: float = 0.1     # per-row relative noise on dxx, dyy
    margin: float = 1.0     # diagonal dominance margin
    adv: float | None = None  # advection; defaults to k


ION = Species(ION_K)
ELECTRON = Species(ELECTRON_K)


def picard_scale(p: int) -> float:
    """Operator scale at Picard step p: sc = 1 + 0.3 * 0.05**p."""
    return 1.0 + 0.3 * (0.05 ** p)


@dataclasses.dataclass
class Batch:
    pattern: Pattern
    g0: int                 # global index of the first system
    values: np.ndarray      # [count, nnz] fp64, CSR order
    b: np.ndarray           # [count, n] fp64

    @property
    def count(self) -> int:
        return self.values.shape[0]


def _species_params(g: np.ndarray, ion: Species, electron: Species):
    is_e = (g % 2) == 1
    def pick(name):
        vi = getattr(ion, name)
        ve = getattr(electron, name)
        if name == "adv":
            vi = ion.k if vi is None else vi
            ve = electron.k if ve is None else ve
        return np.where(is_e, ve, vi).astype(np.float64)
    return {f: pick(f) for f in ("k", "cross", "jitter", "margin", "adv")}


def make_batch(g0: int, count: int, nx: int = 32, ny: int = 31, *,
               seed: int = DEFAULT_SEED, picard: int = 0, scale: float | None = None,
               ion: Species = ION, electron: Species = ELECTRON,
               pattern: Pattern | None = None, chunk: int = 1024,
               threads: int | None = None) -> Batch:
    """Generate systems g0 .. g0+count-1 (CSR values + right-hand sides).

    Row r = (i, j) of system g:
      dxx = k sc (1 + jitter N1), dyy = k sc (1 + jitter N2),
      dxy = cross k sc U(-1, 1)
      ax = adv sc (i - (nx-1)/2)/nx,  ay = adv sc j/ny
      W = -dxx - ax/2, E = -dxx + ax/2, S = -dyy - ay/2, N = -dyy + ay/2
      SW = NE = +dxy/2, NW = SE = -dxy/2
      diagonal = margin + sum |in-grid off-diagonals|   (strict dominance)
      b = exp(-(vpar^2 + vperp^2)/2) + 1e-3, times (1 + 0.01 N3)
    """
    pat = pattern if pattern is not None else stencil_pattern(nx, ny)
    nx, ny, n = pat.nx, pat.ny, pat.n
    sc = picard_scale(picard) if scale is None else float(scale)
    values = np.empty((count, pat.nnz), np.float64)
    b = np.empty((count, n), np.float64)
    r = np.arange(n, dtype=np.int64)
    ii = (r % nx).astype(np.float64)
    jj = (r // nx).astype(np.float64)
    # in-grid mask per neighbour type, [9, n]
    ri, rj = r % nx, r // nx
    mask = np.zeros((9, n), bool)
    for t, (di, dj) in enumerate(STENCIL):
        mask[t] = (ri + di >= 0) & (ri + di < nx) & (rj + dj >= 0) & (rj + dj < ny)
    vpar = np.linspace(-3.0, 3.0, nx)[ri]
    vperp = np.linspace(0.0, 3.0, ny)[rj]
    maxw = np.exp(-(vpar * vpar + vperp * vperp) / 2.0) + 1e-3
    ent_t = pat.ntype.astype(np.int64)
    ent_r = pat.row_of.astype(np.int64)
    def work(c0):
        c1 = min(count, c0 + chunk)
        g = np.arange(g0 + c0, g0 + c1, dtype=np.int64)[:, None]
        P = _species_params(g, ion, electron)
        k = P["k"] * sc
        n1 = normal(seed, g, r[None, :], F_DXX_A, F_DXX_B)
        n2 = normal(seed, g, r[None, :], F_DYY_A, F_DYY_B)
        u = 2.0 * uniform01(seed, g, r[None, :], F_DXY) - 1.0
        dxx = k * (1.0 + P["jitter"] * n1)
        dyy = k * (1.0 + P["jitter"] * n2)
        dxy = P["cross"] * k * u
        ax = P["adv"] * sc * (ii - (nx - 1) / 2.0) / nx
        ay = P["adv"] * sc * jj / ny
        coef = np.empty((9, c1 - c0, n), np.float64)
        coef[0] = dxy / 2.0          # SW
        coef[1] = -dyy - ay / 2.0    # S
        coef[2] = -dxy / 2.0         # SE
        coef[3] = -dxx - ax / 2.0    # W
        coef[5] = -dxx + ax / 2.0    # E
        coef[6] = -dxy / 2.0         # NW
        coef[7] = -dyy + ay / 2.0    # N
        coef[8] = dxy / 2.0          # NE
        diag = np.broadcast_to(P["margin"], (c1 - c0, n)).copy()
        for t in (0, 1, 2, 3, 5, 6, 7, 8):   # fixed order -> chunk-independent
            diag += np.where(mask[t][None, :], np.abs(coef[t]), 0.0)
        coef[CENTER] = diag
        values[c0:c1] = coef[ent_t, :, ent_r].T
        n3 = normal(seed, g, r[None, :], F_B_A, F_B_B)
        b[c0:c1] = maxw[None, :] * (1.0 + 0.01 * n3)

    starts = list(range(0, count, chunk))
    if threads is None:
        threads = min(len(starts), os.cpu_count() or 1, 32)
    if threads <= 1 or len(starts) <= 1:
        for c0 in starts:
            work(c0)
    else:
        with cf.ThreadPoolExecutor(threads) as ex:
            list(ex.map(work, starts))
    return Batch(pat, g0, values, b)


# ---------------------------------------------------------------- layouts --
def ell_width(pat_or_rowptr) -> int:
    rp = pat_or_rowptr.row_ptr if isinstance(pat_or_rowptr, Pattern) else pat_or_rowptr
    return int(np.max(np.diff(np.asarray(rp))))


def ell_layout(row_ptr: np.ndarray, col_idx: np.ndarray, width: int | None = None):
    """ELL layout of a shared CSR pattern.

    Slot k of row i holds the k-th CSR entry of row i; storage is column-major
    (slot k of row i at k*n + i).  Padding slots (rows with fewer entries)
    point at the row itself and carry value 0 (reading R12).
    Returns (ell_col[width*n] int32, src[width*n] int64 CSR entry or -1).
    """
    row_ptr = np.asarray(row_ptr, np.int64)
    n = row_ptr.size - 1
    W = ell_width(row_ptr) if width is None else int(width)
    ell_col = np.empty(W * n, np.int32)
    src = np.full(W * n, -1, np.int64)
    for i in range(n):
        a, e = row_ptr[i], row_ptr[i + 1]
        for k in range(W):
            if a + k < e:
                ell_col[k * n + i] = col_idx[a + k]
                src[k * n + i] = a + k
            else:
                ell_col[k * n + i] = i
    return ell_col, src


def csr_values_to_ell(values: np.ndarray, row_ptr, col_idx, width: int | None = None):
    """[count, nnz] CSR-ordered values -> [count, W*n] ELL column-major values."""
    _, src = ell_layout(row_ptr, col_idx, width)
    out = np.zeros((values.shape[0], src.size), np.float64)
    ok = src >= 0
    out[:, ok] = values[:, src[ok]]
    return out


def random_pattern(n: int, max_row: int, seed: int = 1, density: float = 0.6) -> tuple:
    """A non-stencil shared pattern with a full diagonal and <= max_row
    entries per row, columns sorted; used to prove the kernel is pattern-generic."""
    rng = np.random.default_rng(seed)
    rp = [0]
    cols = []
    for i in range(n):
        m = int(rng.integers(0, max_row)) if n > 1 else 0
        m = min(m, n - 1)
        others = rng.choice(np.delete(np.arange(n), i), size=m, replace=False) if m else []
        row = sorted(set([i, *map(int, others)]))
        cols.extend(row)
        rp.append(len(cols))
    return np.asarray(rp, np.int32), np.asarray(cols, np.int32)


def random_dd_values(row_ptr, col_idx, count: int, seed: int = 2, margin: float = 1.0,
                     offscale: float = 1.0) -> np.ndarray:
    """Strictly diagonally dominant random values on an arbitrary pattern."""
    row_ptr = np.asarray(row_ptr, np.int64)
    n = row_ptr.size - 1
    rng = np.random.default_rng(seed)
    vals = rng.uniform(-offscale, offscale, size=(count, int(row_ptr[-1])))
    for i in range(n):
        a, e = row_ptr[i], row_ptr[i + 1]
        cs = np.asarray(col_idx[a:e])
        d = a + int(np.nonzero(cs == i)[0][0])
        off = np.abs(vals[:, a:e]).sum(axis=1) - np.abs(vals[:, d])
        vals[:, d] = (margin + off) * np.where(rng.random(count) < 0.5, 1.0, -1.0)
    return vals


def random_rhs(count: int, n: int, seed: int = 3) -> np.ndarray:
    return np.random.default_rng(seed).standard_normal((count, n))
