"""Seeded, synthetic workload definitions shared by the oracle and the CUDA path.

This module holds INPUTS only -- none of the method's arithmetic:

* reaction-network specifications as plain data (species, initial microstate
  x0, reactant copy numbers c_k, net change nu_k, intrinsic rates r_k, the
  finite-buffer weights w and cap N).  Turning a specification into microstates
  and rates (propensities, DFS enumeration, P:L37-59 and L81 of
  /root/reference/PAPER.md) is done independently by ``oracle/`` and by the
  library; neither side imports the other.
* the config-5 synthetic banded Markov generator: a
  counter-based splitmix64 stream that emits OFF-DIAGONAL transition rates
  only.  The diagonal (eq. 4) is derived by each side's own ingest.

The readings of the paper's networks (reaction lists, buffer rule, parameter
values) are recorded in DESIGN.md section 3 ("readings") and SURVEY.md App. A.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List

import numpy as np

__all__ = [
    "Network", "birth_death", "toggle_switch", "brusselator", "schnakenberg",
    "schlogl", "cyclic3", "CONFIGS", "config_network", "banded_markov",
    "uniform_start", "random_start", "banded_markov_fast", "build_generator",
]


@dataclass(frozen=True)
class Network:
    """A finitely buffered reaction network (Cao & Liang [17]).

    Reaction k fires from microstate x with propensity
    r_k * prod_i C(x_i, reactants[k][i]) and moves to x + change[k]; it is
    enabled only if the target is non-negative and obeys the buffer
    sum_i weights[i] * x_i <= cap (SURVEY.md App. A reading 7).
    Reactions are listed in the declared order that the DFS enumeration tries.
    """

    name: str
    species: List[str]
    x0: List[int]
    reactants: List[List[int]]
    change: List[List[int]]
    rates: List[float]
    weights: List[int]
    cap: int
    meta: dict = field(default_factory=dict, compare=False)

    @property
    def m(self) -> int:
        return len(self.species)

    @property
    def R(self) -> int:
        return len(self.rates)

    def arrays(self):
        """Plain int32/float64 arrays in the (R, m) layout both enumerators take."""
        return (
            np.asarray(self.x0, dtype=np.int32),
            np.asarray(self.reactants, dtype=np.int32).reshape(self.R, self.m),
            np.asarray(self.change, dtype=np.int32).reshape(self.R, self.m),
            np.asarray(self.rates, dtype=np.float64),
            np.asarray(self.weights, dtype=np.int32),
            int(self.cap),
        )


def birth_death(N: int = 100, lam: float = 10.0, mu: float = 1.0) -> Network:
    """Single species X: R0 0->X (lam), R1 X->0 (mu*x); cap x <= N (config 1)."""
    return Network(
        name=f"birth_death_N{N}", species=["X"], x0=[0],
        reactants=[[0], [1]], change=[[1], [-1]], rates=[lam, mu],
        weights=[1], cap=N, meta={"lam": lam, "mu": mu},
    )


def toggle_switch(N: int = 224, s: float = 50.0, d: float = 1.0, b: float = 0.005,
                  u: float = 0.1) -> Network:
    """Genetic toggle switch with dimer repression (Gardner et al. [16]).

    State (pA, pB, GA, GB, GAb, GBb), x0 = (0,0,1,1,0,0).  Reactions, in the
    declared DFS order:
      R0 GA -> GA + A     (s)          R1 GB -> GB + B     (s)
      R2 A -> 0           (d * pA)     R3 B -> 0           (d * pB)
      R4 GA + 2B -> GAb   (b * C(pB,2))  R5 GAb -> GA + 2B (u)
      R6 GB + 2A -> GBb   (b * C(pA,2))  R7 GBb -> GB + 2A (u)
    Buffer pA + pB + 2 GAb + 2 GBb <= N.  Gives n = 2N^2-2N+4 states.
    """
    #            pA pB GA GB GAb GBb
    reac = [[0, 0, 1, 0, 0, 0],
            [0, 0, 0, 1, 0, 0],
            [1, 0, 0, 0, 0, 0],
            [0, 1, 0, 0, 0, 0],
            [0, 2, 1, 0, 0, 0],
            [0, 0, 0, 0, 1, 0],
            [2, 0, 0, 1, 0, 0],
            [0, 0, 0, 0, 0, 1]]
    chg = [[1, 0, 0, 0, 0, 0],
           [0, 1, 0, 0, 0, 0],
           [-1, 0, 0, 0, 0, 0],
           [0, -1, 0, 0, 0, 0],
           [0, -2, -1, 0, 1, 0],
           [0, 2, 1, 0, -1, 0],
           [-2, 0, 0, -1, 0, 1],
           [2, 0, 0, 1, 0, -1]]
    return Network(
        name=f"toggle_N{N}", species=["pA", "pB", "GA", "GB", "GAb", "GBb"],
        x0=[0, 0, 1, 1, 0, 0], reactants=reac, change=chg,
        rates=[s, s, d, d, b, u, b, u], weights=[1, 1, 0, 0, 2, 2], cap=N,
        meta={"s": s, "d": d, "b": b, "u": u},
    )


def brusselator(N: int = 1000, k0: float = 1.0, k1: float = 1.0, k2: float = 1.0,
                k3: float = 1.0) -> Network:
    """Brusselator [21]: R0 0->X, R1 X->Y, R2 2X+Y->3X, R3 X->0; x+y <= N."""
    return Network(
        name=f"brusselator_N{N}", species=["X", "Y"], x0=[0, 0],
        reactants=[[0, 0], [1, 0], [2, 1], [1, 0]],
        change=[[1, 0], [-1, 1], [1, -1], [-1, 0]],
        rates=[k0, k1, k2, k3], weights=[1, 1], cap=N,
    )


def schnakenberg(N: int = 2000, k1: float = 500.0, k2: float = 1.0, k3: float = 400.0,
                 k4: float = 1.0, k5: float = 1e-6, k6: float | None = None) -> Network:
    """Schnakenberg [23]: R0 0->X, R1 X->0, R2 0->Y, R3 Y->0, R4 2X+Y->3X,
    R5 3X->2X+Y; x+y <= N.  k6 defaults to the detailed-balance value
    3*k5*(k3/k4)/(k1/k2), which gives the product-Poisson law."""
    if k6 is None:
        k6 = 3.0 * k5 * (k3 / k4) / (k1 / k2)
    return Network(
        name=f"schnakenberg_N{N}", species=["X", "Y"], x0=[0, 0],
        reactants=[[0, 0], [1, 0], [0, 0], [0, 1], [2, 1], [3, 0]],
        change=[[1, 0], [-1, 0], [0, 1], [0, -1], [1, -1], [-1, 1]],
        rates=[k1, k2, k3, k4, k5, k6], weights=[1, 1], cap=N,
        meta={"k1": k1, "k2": k2, "k3": k3, "k4": k4, "k5": k5, "k6": k6},
    )


def schlogl(N: int = 700, c1: float = 0.015, c2: float = 6e-5, c3: float = 100.0,
            c4: float = 1.65) -> Network:
    """Schloegl: R0 2X->3X (c1 C(x,2)), R1 3X->2X (c2 C(x,3)), R2 0->X (c3),
    R3 X->0 (c4 x); x <= N.  One-dimensional, so it has a product closed form."""
    return Network(
        name=f"schlogl_N{N}", species=["X"], x0=[0],
        reactants=[[2], [3], [0], [1]], change=[[1], [-1], [1], [-1]],
        rates=[c1, c2, c3, c4], weights=[1], cap=N,
        meta={"c1": c1, "c2": c2, "c3": c3, "c4": c4},
    )


def cyclic3(molecules: int = 3, k: float = 1.0) -> Network:
    """A -> B -> C -> A with a conserved number of molecules: a period-3 chain
    whose undirected state graph has odd cycles."""
    return Network(
        name=f"cyclic3_{molecules}", species=["A", "B", "C"], x0=[molecules, 0, 0],
        reactants=[[1, 0, 0], [0, 1, 0], [0, 0, 1]],
        change=[[-1, 1, 0], [0, -1, 1], [1, 0, -1]],
        rates=[k, k, k], weights=[1, 1, 1], cap=molecules,
    )


# BASELINE.json configs.  omega per reading 1 of SURVEY 8(c6).
CONFIGS = {
    "cfg1_birth_death": dict(network=lambda: birth_death(100, 10.0, 1.0), omega=0.9, tol=1e-12),
    "cfg2_toggle_100k": dict(network=lambda: toggle_switch(224), omega=0.9, tol=1e-12),
    "cfg3a_schnakenberg_2m": dict(network=lambda: schnakenberg(2000), omega=1.0, tol=1e-12),
    "cfg3b_brusselator_2m": dict(network=lambda: brusselator(2000), omega=0.9, tol=1e-12),
    "cfg4_toggle_20m": dict(network=lambda: toggle_switch(3164), omega=0.9, tol=1e-12),
}


def config_network(name: str) -> Network:
    return CONFIGS[name]["network"]()


# Batched sweeps: member b of a sweep over a config scales the
# network's rates by these per-reaction factors (all > 0, so every member has
# the same reachable states and sparsity pattern).
SWEEP_FACTORS = [1.0, 0.7, 1.3, 2.0, 0.5, 1.1, 0.9, 1.6]


def sweep_networks(name: str, batch: int, first: int = 0):
    """`batch` variants of config `name` (sweep members first .. first+batch-1):
    reaction k of member b has rate r_k * SWEEP_FACTORS[b] ** (+1 for even k,
    -0.5 for odd k); member 0 is the configuration itself."""
    base = config_network(name)
    out = []
    for b in range(first, first + batch):
        f = SWEEP_FACTORS[b % len(SWEEP_FACTORS)]
        rates = [r * (f if k % 2 == 0 else f ** -0.5) for k, r in enumerate(base.rates)]
        out.append(Network(name=f"{base.name}_sweep{b}", species=base.species, x0=base.x0,
                           reactants=base.reactants, change=base.change, rates=rates,
                           weights=base.weights, cap=base.cap, meta=dict(base.meta, sweep=b)))
    return out


# ----------------------------------------------------------------------------
# Config 5: synthetic banded Markov generator ("Config 5
# generator").  Counter-based splitmix64; every source state j owns the stream
# seeded with seed ^ (j * 0x9E3779B97F4A7C15).  Off-diagonal rates only.
# ----------------------------------------------------------------------------
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _splitmix_next(state: np.ndarray) -> np.ndarray:
    """Advance each uint64 stream in place and return its next output."""
    with np.errstate(over="ignore"):
        state += _GOLDEN
        z = state.copy()
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _rate_from(r: np.ndarray) -> np.ndarray:
    # 1 + (r >> 11) * 2^-53 : exact doubles in [1, 2)
    return 1.0 + (r >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def banded_markov(n: int, mu: int = 10, width: int = 1024, irregular: bool = False,
                  seed: int = 1):
    """Generate the off-diagonal COO of a config-5 synthetic banded generator.

    Per source state j (column j): always j -> j-1 and j -> j+1 (when in
    range), then m_j more targets i = j + delta, delta uniform on
    [-width, width] minus {-1, 0, 1}, rejecting out-of-range and duplicate
    targets; m_j = mu-3 (const) or uniform on [0, 2(mu-3)] (irregular).
    Returns (row=int32 target i, col=int32 source j, rate=float64) sorted by
    column then emission order.  Bit-reproducible for a given seed.
    """
    if n < 2 or mu < 3 or width < 2:
        raise ValueError("banded_markov needs n >= 2, mu >= 3, width >= 2")
    width = min(width, n)
    j = np.arange(n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        st = np.uint64(seed) ^ (j * _GOLDEN)
    extra = mu - 3
    if irregular:
        m_j = (_splitmix_next(st) % np.uint64(2 * extra + 1)).astype(np.int64)
    else:
        m_j = np.full(n, extra, dtype=np.int64)
    cap_slots = 2 + (2 * extra if irregular else extra)
    tgt = np.full((n, cap_slots), -1, dtype=np.int64)
    rate = np.zeros((n, cap_slots), dtype=np.float64)
    cnt = np.zeros(n, dtype=np.int64)
    ji = j.astype(np.int64)
    for off in (-1, 1):
        ok = (ji + off >= 0) & (ji + off < n)
        r = np.zeros(n, dtype=np.uint64)
        sub = st[ok]
        r_ok = _splitmix_next(sub)
        st[ok] = sub
        r[ok] = r_ok
        idx = np.nonzero(ok)[0]
        tgt[idx, cnt[idx]] = ji[idx] + off
        rate[idx, cnt[idx]] = _rate_from(r[idx])
        cnt[idx] += 1
    want = cnt + m_j
    attempts = np.zeros(n, dtype=np.int64)
    max_attempts = 64 * np.maximum(m_j, 1)
    span = np.uint64(2 * width - 2)
    active = np.nonzero((cnt < want) & (attempts < max_attempts))[0]
    while active.size:
        sub = st[active]
        r = _splitmix_next(sub)
        st[active] = sub
        attempts[active] += 1
        k = (r % span).astype(np.int64)
        delta = np.where(k < width - 1, -width + k, 2 + (k - (width - 1)))
        cand = ji[active] + delta
        ok = (cand >= 0) & (cand < n)
        ok &= ~(tgt[active] == cand[:, None]).any(axis=1)
        acc = active[ok]
        if acc.size:
            sub = st[acc]
            rr = _splitmix_next(sub)
            st[acc] = sub
            tgt[acc, cnt[acc]] = cand[ok]
            rate[acc, cnt[acc]] = _rate_from(rr)
            cnt[acc] += 1
        active = active[(cnt[active] < want[active]) & (attempts[active] < max_attempts[active])]
    mask = tgt >= 0
    cols = np.broadcast_to(ji[:, None], tgt.shape)[mask].astype(np.int32)
    rows = tgt[mask].astype(np.int32)
    return rows, cols, rate[mask]


def uniform_start(n: int) -> np.ndarray:
    return np.full(n, 1.0 / n)


def random_start(n: int, seed: int = 0) -> np.ndarray:
    """A strictly positive seeded start vector (not normalised)."""
    g = np.random.default_rng(seed)
    return g.random(n) + 0.5


# ----------------------------------------------------------------------------
# The same config-5 generator in C (workloads/banded_markov.c, OpenMP over
# source states) for the 1M-100M-row sweep; tests/test_workloads.py checks it
# against banded_markov above array for array.
# ----------------------------------------------------------------------------
import ctypes as _C  # noqa: E402
import os as _os  # noqa: E402
import subprocess as _sp  # noqa: E402

_HERE = _os.path.dirname(_os.path.abspath(__file__))
_GEN_SRC = _os.path.join(_HERE, "banded_markov.c")
_GEN_LIB = _os.path.join(_HERE, "libwl_gen.so")
_gen = None


def build_generator(force: bool = False) -> str:
    """Compile libwl_gen.so (gcc, OpenMP; input generation only)."""
    import hashlib
    with open(_GEN_SRC, "rb") as f:
        digest = hashlib.sha256(f.read()).hexdigest()   # rebuild on any source change (not mtimes)
    stamp = _GEN_LIB + ".sha256"
    if force or not _os.path.exists(_GEN_LIB) or not _os.path.exists(stamp) or open(stamp).read().strip() != digest:
        tmp = _GEN_LIB + f".tmp{_os.getpid()}"
        _sp.check_call(["gcc", "-O2", "-std=c99", "-fopenmp", "-fPIC", "-shared", "-Wall", "-o", tmp, _GEN_SRC])
        _os.replace(tmp, _GEN_LIB)
        with open(stamp, "w") as f:
            f.write(digest + "\n")
    return _GEN_LIB


def banded_markov_fast(n: int, mu: int = 10, width: int = 1024, irregular: bool = False, seed: int = 1):
    """banded_markov(...) computed by the C generator: identical arrays."""
    global _gen
    if n < 2 or mu < 3 or width < 2:
        raise ValueError("banded_markov needs n >= 2, mu >= 3, width >= 2")
    if _gen is None:
        L = _C.CDLL(build_generator())
        i64p = _C.POINTER(_C.c_int64)
        L.wl_banded_markov_count.restype = _C.c_int64
        L.wl_banded_markov_count.argtypes = [_C.c_int64, _C.c_int, _C.c_int64, _C.c_int, _C.c_uint64, i64p]
        L.wl_banded_markov_fill.restype = None
        L.wl_banded_markov_fill.argtypes = [_C.c_int64, _C.c_int, _C.c_int64, _C.c_int, _C.c_uint64, i64p,
                                            _C.POINTER(_C.c_int32), _C.POINTER(_C.c_int32),
                                            _C.POINTER(_C.c_double)]
        _gen = L
    off = np.empty(n + 1, dtype=np.int64)
    args = (n, mu, width, 1 if irregular else 0, seed)
    nnz = _gen.wl_banded_markov_count(*args, off.ctypes.data_as(_C.POINTER(_C.c_int64)))
    if nnz < 0:
        raise ValueError("wl_banded_markov_count: bad arguments")
    rows = np.empty(nnz, dtype=np.int32)
    cols = np.empty(nnz, dtype=np.int32)
    rates = np.empty(nnz, dtype=np.float64)
    _gen.wl_banded_markov_fill(*args, off.ctypes.data_as(_C.POINTER(_C.c_int64)),
                               rows.ctypes.data_as(_C.POINTER(_C.c_int32)),
                               cols.ctypes.data_as(_C.POINTER(_C.c_int32)),
                               rates.ctypes.data_as(_C.POINTER(_C.c_double)))
    return rows, cols, rates
