"""CPU oracle for the CME steady-state Jacobi hot path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It is a
ctypes wrapper around ``cme_oracle.c`` (plain C99, optional OpenMP), which is
written from /root/reference/PAPER.md and the readings in DESIGN.md section 3
and shares no code with the CUDA library.

Pins (tests/test_oracle_*.py) tie every function to something other than
itself: Table I statistics, closed-form steady states (truncated
Poisson, product-Poisson Schnakenberg, Schloegl), numpy/LAPACK solves, brute
force on tiny graphs, and structural invariants.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cme_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

STATUS = {0: "OK", 1: "INVALID_ARG", 2: "NEGATIVE_RATE", 3: "ZERO_OUTFLOW", 5: "OOM",
          8: "NOT_CONVERGED", 9: "STAGNATED", 10: "NUMERIC"}


class OracleError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: {STATUS.get(code, code)}")
        self.code = code


def _src_hash() -> str:
    """sha256 of the oracle's C source and header (rebuild on any change; mtimes
    are not trusted)."""
    import hashlib
    h = hashlib.sha256()
    for p in (_SRC, os.path.join(_HERE, "cme_oracle.h")):
        with open(p, "rb") as f:
            h.update(f.read())
    return h.hexdigest()


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (no CUDA)."""
    digest = _src_hash()
    stamp = _LIB + ".sha256"
    if force or not os.path.exists(_LIB) or not os.path.exists(stamp) or open(stamp).read().strip() != digest:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fopenmp", "-fPIC", "-shared",
                               "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
        with open(stamp, "w") as f:
            f.write(digest + "\n")
    return _LIB


_lib = None
_p = C.POINTER
i32p, i64p, f64p = _p(C.c_int32), _p(C.c_int64), _p(C.c_double)


class _Packed(C.Structure):
    _fields_ = [("n", C.c_int64), ("n_slots", C.c_int64), ("n_slices", C.c_int64),
                ("n_ell", C.c_int64), ("band_on", C.c_int32), ("window", C.c_int32),
                ("lo", f64p), ("up", f64p), ("inv_d", f64p), ("row_of", i32p),
                ("slice_off", i64p), ("slice_w", i32p), ("val", f64p), ("col", i32p)]


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        L.oracle_free.argtypes = [C.c_void_p]
        L.oracle_enumerate.argtypes = [C.c_int, i32p, C.c_int, i32p, i32p, f64p, i32p, C.c_int64,
                                       i64p, i64p, _p(i32p), _p(i32p), _p(i32p), _p(f64p)]
        L.oracle_ingest.argtypes = [C.c_int64, C.c_int64, i32p, i32p, f64p, C.c_int,
                                    _p(i64p), _p(i32p), _p(f64p), _p(f64p)]
        L.oracle_order_dfs.argtypes = [C.c_int64, i64p, i32p, C.c_int64, i32p]
        L.oracle_order_rcm.argtypes = [C.c_int64, i64p, i32p, i32p]
        L.oracle_permute.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, i32p,
                                     _p(i64p), _p(i32p), _p(f64p), _p(f64p)]
        L.oracle_period.argtypes = [C.c_int64, i64p, i32p, C.c_int64]
        L.oracle_period.restype = C.c_int64
        L.oracle_pack.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, C.c_int32, C.c_int32,
                                  C.c_int32, _p(_Packed)]
        L.oracle_packed_free.argtypes = [_p(_Packed)]
        L.oracle_jacobi_step.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, C.c_double, f64p, f64p]
        L.oracle_jacobi_solve.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, f64p, C.c_double,
                                          C.c_double, C.c_int64, C.c_int64, C.c_int, C.c_double,
                                          C.c_int, f64p, i64p, f64p, f64p]
        L.oracle_lu_steady.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, f64p]
        L.oracle_transient.argtypes = [C.c_int64, i64p, i32p, f64p, f64p, f64p, C.c_double, C.c_double,
                                       f64p, i64p, f64p]
        _lib = L
    return _lib


def _ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def _take(ptr, n, dtype):
    """Copy a malloc()ed C array into numpy and free it."""
    if n == 0:
        out = np.zeros(0, dtype=dtype)
    else:
        out = np.ctypeslib.as_array(ptr, shape=(n,)).astype(dtype, copy=True)
    lib().oracle_free(C.cast(ptr, C.c_void_p))
    return out


def _check(rc, what):
    if rc != 0:
        raise OracleError(rc, what)


@dataclass
class CSR:
    """Off-diagonal part of A by rows (row i <- col j: transition j -> i) + diagonal."""
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    diag: np.ndarray

    @property
    def nnz_offdiag(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def nnz(self) -> int:
        """nnz(A) including the diagonal (Table I convention)."""
        return self.nnz_offdiag + self.n

    def _a(self):
        return (_ptr(self.row_ptr, i64p), _ptr(self.col, i32p), _ptr(self.val, f64p),
                _ptr(self.diag, f64p))

    def dense(self) -> np.ndarray:
        A = np.zeros((self.n, self.n))
        for i in range(self.n):
            s, e = self.row_ptr[i], self.row_ptr[i + 1]
            A[i, self.col[s:e]] = self.val[s:e]
            A[i, i] = self.diag[i]
        return A


def enumerate_network(net):
    """Return (states[n, m], row, col, rate) of the off-diagonal COO."""
    x0, reac, chg, rates, w, cap = net.arrays()
    reac = np.ascontiguousarray(reac); chg = np.ascontiguousarray(chg)
    n, nnz = C.c_int64(), C.c_int64()
    S, Rr, Cc, V = i32p(), i32p(), i32p(), f64p()
    rc = lib().oracle_enumerate(net.m, _ptr(x0, i32p), net.R, _ptr(reac, i32p), _ptr(chg, i32p),
                                _ptr(rates, f64p), _ptr(w, i32p), cap, C.byref(n), C.byref(nnz),
                                C.byref(S), C.byref(Rr), C.byref(Cc), C.byref(V))
    _check(rc, "oracle_enumerate")
    states = _take(S, n.value * net.m, np.int32).reshape(n.value, net.m)
    return states, _take(Rr, nnz.value, np.int32), _take(Cc, nnz.value, np.int32), \
        _take(V, nnz.value, np.float64)


def ingest(n, row, col, rate, diag_given=False) -> CSR:
    row = np.ascontiguousarray(row, dtype=np.int32)
    col = np.ascontiguousarray(col, dtype=np.int32)
    rate = np.ascontiguousarray(rate, dtype=np.float64)
    rp, cj, vv, d = i64p(), i32p(), f64p(), f64p()
    rc = lib().oracle_ingest(n, len(row), _ptr(row, i32p), _ptr(col, i32p), _ptr(rate, f64p),
                             int(diag_given), C.byref(rp), C.byref(cj), C.byref(vv), C.byref(d))
    _check(rc, "oracle_ingest")
    row_ptr = _take(rp, n + 1, np.int64)
    nz = int(row_ptr[-1])
    return CSR(n, row_ptr, _take(cj, nz, np.int32), _take(vv, nz, np.float64), _take(d, n, np.float64))


def network_csr(net) -> CSR:
    states, r, c, v = enumerate_network(net)
    return ingest(len(states), r, c, v)


def order_dfs(A: CSR, root: int = 0) -> np.ndarray:
    p = np.empty(A.n, dtype=np.int32)
    _check(lib().oracle_order_dfs(A.n, _ptr(A.row_ptr, i64p), _ptr(A.col, i32p), root, _ptr(p, i32p)),
           "oracle_order_dfs")
    return p


def order_rcm(A: CSR) -> np.ndarray:
    p = np.empty(A.n, dtype=np.int32)
    _check(lib().oracle_order_rcm(A.n, _ptr(A.row_ptr, i64p), _ptr(A.col, i32p), _ptr(p, i32p)),
           "oracle_order_rcm")
    return p


def permute(A: CSR, new_to_old: np.ndarray) -> CSR:
    new_to_old = np.ascontiguousarray(new_to_old, dtype=np.int32)
    rp, cj, vv, d = i64p(), i32p(), f64p(), f64p()
    _check(lib().oracle_permute(A.n, *A._a(), _ptr(new_to_old, i32p), C.byref(rp), C.byref(cj),
                                C.byref(vv), C.byref(d)), "oracle_permute")
    row_ptr = _take(rp, A.n + 1, np.int64)
    nz = int(row_ptr[-1])
    return CSR(A.n, row_ptr, _take(cj, nz, np.int32), _take(vv, nz, np.float64),
               _take(d, A.n, np.float64))


def period(A: CSR, root: int = 0) -> int:
    return int(lib().oracle_period(A.n, _ptr(A.row_ptr, i64p), _ptr(A.col, i32p), root))


BAND = {"auto": 0, "always": 1, "never": 2}


def pack(A: CSR, window: int = 256, band: str = "auto", uniform: bool = False, group: int = 1) -> dict:
    """Layout v0 arrays of an already-ordered matrix.
    group = slices sharing a width (1 warp-grained, 8 block-sliced); uniform = plain ELL."""
    P = _Packed()
    _check(lib().oracle_pack(A.n, *A._a(), window, BAND[band], 0 if uniform else group, C.byref(P)),
           "oracle_pack")
    try:
        def cp(ptr, k, dt):
            return np.ctypeslib.as_array(ptr, shape=(k,)).astype(dt, copy=True) if k else np.zeros(0, dt)
        out = dict(n=P.n, n_slots=P.n_slots, n_slices=P.n_slices, n_ell=P.n_ell,
                   band_on=bool(P.band_on), window=P.window,
                   lo=cp(P.lo, P.n_slots, np.float64), up=cp(P.up, P.n_slots, np.float64),
                   inv_d=cp(P.inv_d, P.n_slots, np.float64), row_of=cp(P.row_of, P.n_slots, np.int32),
                   slice_off=cp(P.slice_off, P.n_slices + 1, np.int64),
                   slice_w=cp(P.slice_w, P.n_slices, np.int32),
                   val=cp(P.val, P.n_ell, np.float64), col=cp(P.col, P.n_ell, np.int32))
    finally:
        lib().oracle_packed_free(C.byref(P))
    return out


def compact(A: CSR, P: dict):
    """Compact encoding of a layout-v0 pack P = pack(A, ...)
    of the already-ordered matrix A, from its definition: the stored rows are
    those of M = |D|^-1 O, the Jacobi iteration matrix of P:L111 eq. 8
    (x_i <- sum_{j!=i} a_ij x_j / (-a_ii)), i.e. val_c[e] = a_rj / (-a_rr)
    for the entry e of row r (one IEEE division), lo/up likewise; col16[e] =
    j - r; row8[s] = r - (s // window) * window.  Pad entries and pad slots
    hold 0.  Returns None when the encoding does not apply (window not a power
    of two <= 256, or some |j - r| > 32767)."""
    n, W = P["n"], P["window"]
    if W > 1 and (W > 256 or W & (W - 1)):
        return None
    q_of_e = np.repeat(np.arange(P["n_slices"], dtype=np.int64), 32 * P["slice_w"].astype(np.int64))
    lane = (np.arange(P["n_ell"], dtype=np.int64) - P["slice_off"][q_of_e]) % 32
    slot = 32 * q_of_e + lane                      # slot of every stored entry
    real = slot < n
    row = np.where(real, P["row_of"][np.minimum(slot, P["n_slots"] - 1)], 0).astype(np.int64)
    dneg = -A.diag[row]                            # -a_rr of the entry's row
    delta = np.where(real, P["col"].astype(np.int64) - row, 0)
    if delta.size and np.abs(delta).max() > 32767:
        return None
    val = np.where(real, P["val"] / np.where(real, dneg, 1.0), 0.0)
    out = dict(val=val, col16=delta.astype(np.int16),
               win_shift=int(W).bit_length() - 1 if W > 1 else 0)
    srow = P["row_of"][:n].astype(np.int64)
    if W > 1:
        r8 = np.zeros(P["n_slots"], np.uint8)
        r8[:n] = (srow - (np.arange(n) // W) * W).astype(np.uint8)
        out["row8"] = r8
    if P["band_on"]:
        for k in ("lo", "up"):
            v = np.zeros(P["n_slots"])
            v[:n] = P[k][:n] / (-A.diag[srow])
            out[k] = v
    return out


def value_index(P: dict):
    """Value-indexed form (the CSR-VI idea) of a layout-v0
    pack P: dict = the distinct stored values of P's val (every entry, pads
    included) and, band on, lo/up, ascending; vidx / loi / upi = positions
    in dict.  For a batch (P["batch"] = B > 1, member-minor values) the
    distinct B-tuples in lexicographic order, flattened member-minor.  None
    when there are more than 65536 distinct values (tuples)."""
    B = P.get("batch", 1)
    if B == 1:
        parts = [P["val"]] + ([P["lo"], P["up"]] if P["band_on"] else [])
        d = np.unique(np.concatenate(parts))
        if len(d) > 65536:
            return None
        out = dict(dict=d, vidx=np.searchsorted(d, P["val"]).astype(np.uint16))
        if P["band_on"]:
            out["loi"] = np.searchsorted(d, P["lo"]).astype(np.uint16)
            out["upi"] = np.searchsorted(d, P["up"]).astype(np.uint16)
        return out
    # a batch (B rate sets on one pattern, member-minor values): the distinct
    # B-tuples, lexicographically ascending, and each entry's tuple index
    parts = [P["val"].reshape(-1, B)] + ([P["lo"].reshape(-1, B), P["up"].reshape(-1, B)] if P["band_on"] else [])
    d, inv = np.unique(np.concatenate(parts), axis=0, return_inverse=True)
    if len(d) > 65536:
        return None
    inv = inv.reshape(-1).astype(np.uint16)
    ne = len(parts[0])
    out = dict(dict=d.reshape(-1), vidx=inv[:ne])
    if P["band_on"]:
        ns = len(parts[1])
        out["loi"], out["upi"] = inv[ne:ne + ns], inv[ne + ns:]
    return out


def jacobi_step(A: CSR, x: np.ndarray, omega: float = 1.0) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.empty(A.n)
    _check(lib().oracle_jacobi_step(A.n, *A._a(), omega, _ptr(x, f64p), _ptr(y, f64p)),
           "oracle_jacobi_step")
    return y


@dataclass
class SolveResult:
    p: np.ndarray
    iters: int
    status: str
    delta: float
    resid: float


def jacobi_solve(A: CSR, p0=None, omega=1.0, tol=1e-12, check_every=100, max_iter=1_000_000,
                 stop_mode=0, stag_tol=1e-10, nthreads=1) -> SolveResult:
    p = np.empty(A.n)
    it, de, rs = C.c_int64(), C.c_double(), C.c_double()
    p0p = None
    if p0 is not None:
        p0 = np.ascontiguousarray(p0, dtype=np.float64)
        p0p = _ptr(p0, f64p)
    rc = lib().oracle_jacobi_solve(A.n, *A._a(), p0p, omega, tol, check_every, max_iter, stop_mode,
                                   stag_tol, nthreads, _ptr(p, f64p), C.byref(it), C.byref(de),
                                   C.byref(rs))
    if rc not in (0, 8, 9, 10):
        raise OracleError(rc, "oracle_jacobi_solve")
    return SolveResult(p, it.value, {0: "CONVERGED", 8: "NOT_CONVERGED", 9: "STAGNATED",
                                     10: "NUMERIC"}[rc], de.value, rs.value)


def lu_steady(A: CSR) -> np.ndarray:
    p = np.empty(A.n)
    _check(lib().oracle_lu_steady(A.n, *A._a(), _ptr(p, f64p)), "oracle_lu_steady")
    return p


def transient(A: CSR, t: float, p0=None, eps: float = 1e-14):
    """p(t) = exp(A t) p0 by uniformization; returns (p, terms, Lambda)."""
    p = np.empty(A.n)
    terms, lam = C.c_int64(), C.c_double()
    p0p = None
    if p0 is not None:
        p0 = np.ascontiguousarray(p0, dtype=np.float64)
        p0p = _ptr(p0, f64p)
    _check(lib().oracle_transient(A.n, *A._a(), p0p, t, eps, _ptr(p, f64p), C.byref(terms), C.byref(lam)),
           "oracle_transient")
    return p, terms.value, lam.value
