"""Thin Python binding of libcme (include/cme.h) -- argument marshalling only.

Every step of the CME steady-state path (ingest, reorder, pack, the fused
Jacobi kernels, checks, halo exchange) runs inside libcme.so; this module only
turns numpy arrays / torch tensors into pointers and cme_status codes into
exceptions.  There is no Python or CPU fallback: if libcme.so is missing the
import fails.  Function names are the C names (cme_*).

Vectors may be numpy arrays (host) or torch tensors (host or CUDA); all
vectors are in ORIGINAL state order.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# CME_LIBRARY: load another build of libcme.so (kernel A/B experiments in tools/)
LIB_PATH = os.environ.get("CME_LIBRARY") or os.path.join(_HERE, "libcme.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python paper_conf_ipps_maggionibl13_b200/build.py` "
                      "(nvcc, sm_100a).  There is no fallback path.")

_lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)

# ---- constants (include/cme.h) ---------------------------------------------------------
CME_OK, CME_ERR_INVALID_ARG, CME_ERR_NEGATIVE_RATE, CME_ERR_ZERO_OUTFLOW = 0, 1, 2, 3
CME_ERR_BAD_STATE, CME_ERR_OOM, CME_ERR_CUDA, CME_ERR_NCCL = 4, 5, 6, 7
CME_NOT_CONVERGED, CME_STAGNATED, CME_ERR_NUMERIC, CME_ERR_NO_DEVICE = 8, 9, 10, 11
CME_ERR_TIMEOUT = 12
CME_DIAG_FROM_COLSUMS, CME_DIAG_GIVEN = 0, 1
CME_ORDER_NONE, CME_ORDER_DFS, CME_ORDER_RCM = 0, 1, 2
CME_FMT_DIAG_SELL, CME_FMT_ELL, CME_FMT_CSR, CME_FMT_SELL256 = 0, 1, 2, 3
CME_BAND_AUTO, CME_BAND_ALWAYS, CME_BAND_NEVER = 0, 1, 2
CME_DEVICE_HOST_ONLY = -2
CME_STOP_DELTA_L1, CME_STOP_PAPER_RESID = 0, 1
SOLVE_STATUS = {CME_OK: "CONVERGED", CME_NOT_CONVERGED: "NOT_CONVERGED",
                CME_STAGNATED: "STAGNATED", CME_ERR_NUMERIC: "NUMERIC"}

_p = C.POINTER
i32p, i64p, f64p, u8p, vp = _p(C.c_int32), _p(C.c_int64), _p(C.c_double), _p(C.c_uint8), C.c_void_p


class cme_pack_opts(C.Structure):
    _fields_ = [("slice", C.c_int32), ("window", C.c_int32), ("band", C.c_int32), ("device", C.c_int32)]


class cme_solver_opts(C.Structure):
    _fields_ = [("omega", C.c_double), ("check_every", C.c_int64), ("stop", C.c_int32),
                ("stag_tol", C.c_double), ("stream", C.c_void_p)]


class cme_report(C.Structure):
    _fields_ = [("status", C.c_int32), ("iters", C.c_int64), ("delta", C.c_double),
                ("resid", C.c_double), ("mass", C.c_double), ("omega", C.c_double),
                ("seconds", C.c_double)]


class cme_info(C.Structure):
    _fields_ = [("n", C.c_int64), ("nnz", C.c_int64), ("nnz_offdiag", C.c_int64),
                ("bandwidth", C.c_int64), ("band_density", C.c_double),
                ("band_density3", C.c_double), ("ell_efficiency", C.c_double),
                ("format", C.c_int32), ("order", C.c_int32), ("band_on", C.c_int32),
                ("window", C.c_int32), ("period", C.c_int64), ("norm_inf", C.c_double),
                ("omega", C.c_double), ("n_slots", C.c_int64), ("n_slices", C.c_int64),
                ("n_ell", C.c_int64), ("packed_bytes", C.c_int64), ("bytes_alg", C.c_int64),
                ("bytes_fmt", C.c_int64), ("rank", C.c_int32), ("nranks", C.c_int32),
                ("row_begin", C.c_int64), ("row_end", C.c_int64), ("halo_begin", C.c_int64),
                ("halo_end", C.c_int64), ("kernel", C.c_int32), ("tma_warps", C.c_int32),
                ("tma_stages", C.c_int32), ("grid", C.c_int32), ("batch", C.c_int32),
                ("compact", C.c_int32), ("records", C.c_int32),
                ("wf_steps", C.c_int32), ("wf_lag", C.c_int32), ("halo_fused", C.c_int32),
                ("xwin_kb", C.c_int32)]


class cme_packed_view(C.Structure):
    _fields_ = [("n", C.c_int64), ("n_slots", C.c_int64), ("n_slices", C.c_int64),
                ("n_ell", C.c_int64), ("band_on", C.c_int32), ("window", C.c_int32),
                ("batch", C.c_int32), ("pad_", C.c_int32), ("lo", f64p), ("up", f64p), ("inv_d", f64p), ("row_of", i32p),
                ("slice_off", i64p), ("slice_w", i32p), ("val", f64p), ("col", i32p),
                ("csr_row_ptr", i64p)]


class cme_compact_view(C.Structure):
    _fields_ = [("n", C.c_int64), ("n_slots", C.c_int64), ("n_slices", C.c_int64),
                ("n_ell", C.c_int64), ("band_on", C.c_int32), ("win_shift", C.c_int32),
                ("val", f64p), ("col16", C.POINTER(C.c_int16)), ("row8", C.POINTER(C.c_uint8)),
                ("lo", f64p), ("up", f64p), ("n_dict", C.c_int64), ("dict", f64p),
                ("vidx", C.POINTER(C.c_uint16)), ("loi", C.POINTER(C.c_uint16)), ("upi", C.POINTER(C.c_uint16)),
                ("batch", C.c_int32), ("pad_", C.c_int32)]


class cme_halo_view(C.Structure):
    _fields_ = [("nranks", C.c_int32), ("rank", C.c_int32), ("row_begin", i64p), ("span", i64p),
                ("n_send", C.c_int32), ("n_recv", C.c_int32),
                ("send_peer", i32p), ("send_off", i64p), ("send_cnt", i64p),
                ("recv_peer", i32p), ("recv_off", i64p), ("recv_cnt", i64p)]


_SIGS = {
    "cme_matrix_create_coo": [C.c_int64, C.c_int64, i32p, i32p, f64p, C.c_uint32, _p(vp)],
    "cme_matrix_create_csr": [C.c_int64, i64p, i32p, f64p, C.c_uint32, _p(vp)],
    "cme_matrix_create_coo_batch": [C.c_int64, C.c_int64, i32p, i32p, f64p, C.c_int32, C.c_uint32, _p(vp)],
    "cme_get_batch_report": [vp, _p(cme_report), C.c_int32],
    "cme_reorder": [vp, C.c_int, C.c_int64],
    "cme_set_permutation": [vp, i32p],
    "cme_pack": [vp, C.c_int, _p(cme_pack_opts)],
    "cme_set_solver_opts": [vp, _p(cme_solver_opts)],
    "cme_jacobi_solve": [vp, vp, C.c_double, C.c_int64, vp, i64p],
    "cme_get_report": [vp, _p(cme_report)],
    "cme_transient": [vp, vp, C.c_double, C.c_double, vp, i64p],
    "cme_spmv": [vp, vp, vp],
    "cme_solver_load": [vp, vp],
    "cme_solver_run": [vp, C.c_int64],
    "cme_solver_fetch": [vp, vp],
    "cme_get_info": [vp, _p(cme_info)],
    "cme_get_permutation": [vp, i32p],
    "cme_export_packed": [vp, _p(cme_packed_view)],
    "cme_period": [vp, C.c_int64, i64p],
    "cme_export_xw_plan": [vp, C.c_int32, C.c_int32, C.c_int64, i32p, i64p, i64p],
    "cme_export_compact": [vp, _p(cme_compact_view)],
    "cme_comm_unique_id": [u8p],
    "cme_comm_init": [C.c_int, C.c_int, u8p, C.c_int, _p(vp)],
    "cme_comm_init_local": [C.c_int, i32p, _p(vp)],
    "cme_comm_init_ipc": [C.c_int, C.c_int, C.c_int, _p(vp)],
    "cme_matrix_ipc_export": [vp, u8p],
    "cme_matrix_ipc_attach": [vp, u8p],
    "cme_matrix_plan_partition": [vp, C.c_int, C.c_int],
    "cme_matrix_distribute": [vp, vp],
    "cme_export_halo": [vp, _p(cme_halo_view)],
    "cme_network_enumerate": [C.c_int, i32p, C.c_int, i32p, i32p, f64p, i32p, C.c_int64, _p(vp)],
    "cme_network_enumerate_gpu": [C.c_int, i32p, C.c_int, i32p, i32p, f64p, i32p, C.c_int64, C.c_int, _p(vp)],
    "cme_coo_get": [vp, i64p, i64p, i32p, _p(i32p), _p(i32p), _p(i32p), _p(f64p)],
}
for _name, _args in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = C.c_int
_lib.cme_matrix_destroy.argtypes = [vp]
_lib.cme_matrix_destroy.restype = None
_lib.cme_comm_destroy.argtypes = [vp]
_lib.cme_comm_destroy.restype = None
_lib.cme_coo_destroy.argtypes = [vp]
_lib.cme_coo_destroy.restype = None
_lib.cme_status_string.argtypes = [C.c_int]
_lib.cme_status_string.restype = C.c_char_p
_lib.cme_last_error.restype = C.c_char_p
_lib.cme_abi_version.restype = C.c_int

#: every symbol include/cme.h declares (checked by tests/test_abi.py)
ABI_SYMBOLS = sorted(list(_SIGS) + ["cme_matrix_destroy", "cme_comm_destroy", "cme_coo_destroy",
                                    "cme_status_string", "cme_last_error", "cme_abi_version"])


class CmeError(RuntimeError):
    def __init__(self, status: int, where: str):
        detail = _lib.cme_last_error().decode(errors="replace")
        super().__init__(f"{where}: {_lib.cme_status_string(status).decode()} {detail}".strip())
        self.status = status


def _chk(st: int, where: str, ok=(CME_OK,)):
    if st not in ok:
        raise CmeError(st, where)
    return st


def _vec_ptr(x, n: int, writable: bool = False):
    """Pointer to n contiguous float64 values of a numpy array or torch tensor."""
    if x is None:
        return None, None
    if isinstance(x, np.ndarray):
        if x.dtype != np.float64 or not x.flags.c_contiguous or x.size != n:
            raise ValueError(f"need a contiguous float64 array of {n} values")
        if writable and not x.flags.writeable:
            raise ValueError("output array is read-only")
        return C.c_void_p(x.ctypes.data), x
    import torch
    if isinstance(x, torch.Tensor):
        if x.dtype != torch.float64 or not x.is_contiguous() or x.numel() != n:
            raise ValueError(f"need a contiguous float64 tensor of {n} values")
        return C.c_void_p(x.data_ptr()), x
    raise TypeError("vectors must be numpy arrays or torch tensors")


def _arr(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


# ---- thin wrappers with the C names ------------------------------------------------------
def cme_matrix_create_coo(n, row, col, rate, flags=CME_DIAG_FROM_COLSUMS):
    row, col, rate = _arr(row, np.int32), _arr(col, np.int32), _arr(rate, np.float64)
    h = vp()
    _chk(_lib.cme_matrix_create_coo(n, len(row), row.ctypes.data_as(i32p), col.ctypes.data_as(i32p),
                                    rate.ctypes.data_as(f64p), flags, C.byref(h)), "cme_matrix_create_coo")
    return h


def cme_matrix_create_coo_batch(n, row, col, rates, flags=CME_DIAG_FROM_COLSUMS):
    """rates: array (batch, nnz) -- one rate set per member on the (row, col) pattern."""
    row, col = _arr(row, np.int32), _arr(col, np.int32)
    rates = np.ascontiguousarray(rates, dtype=np.float64)
    if rates.ndim != 2 or rates.shape[1] != len(row):
        raise ValueError("rates must be (batch, nnz)")
    h = vp()
    _chk(_lib.cme_matrix_create_coo_batch(n, len(row), row.ctypes.data_as(i32p), col.ctypes.data_as(i32p),
                                          rates.ctypes.data_as(f64p), rates.shape[0], flags, C.byref(h)),
         "cme_matrix_create_coo_batch")
    return h


def cme_get_batch_report(h, count):
    arr = (cme_report * count)()
    _chk(_lib.cme_get_batch_report(h, arr, count), "cme_get_batch_report")
    return list(arr)


def cme_matrix_create_csr(n, row_ptr, col, rate, flags=CME_DIAG_FROM_COLSUMS):
    row_ptr, col, rate = _arr(row_ptr, np.int64), _arr(col, np.int32), _arr(rate, np.float64)
    h = vp()
    _chk(_lib.cme_matrix_create_csr(n, row_ptr.ctypes.data_as(i64p), col.ctypes.data_as(i32p),
                                    rate.ctypes.data_as(f64p), flags, C.byref(h)), "cme_matrix_create_csr")
    return h


def cme_reorder(h, method=CME_ORDER_NONE, root=0):
    _chk(_lib.cme_reorder(h, method, root), "cme_reorder")


def cme_set_permutation(h, new_to_old):
    p = _arr(new_to_old, np.int32)
    _chk(_lib.cme_set_permutation(h, p.ctypes.data_as(i32p)), "cme_set_permutation")


def cme_pack(h, fmt=CME_FMT_DIAG_SELL, window=256, band=CME_BAND_AUTO, device=-1):
    o = cme_pack_opts(32, window, band, device)
    _chk(_lib.cme_pack(h, fmt, C.byref(o)), "cme_pack")


def cme_set_solver_opts(h, omega=0.0, check_every=100, stop=CME_STOP_DELTA_L1, stag_tol=1e-10, stream=None):
    o = cme_solver_opts(omega, check_every, stop, stag_tol, stream)
    _chk(_lib.cme_set_solver_opts(h, C.byref(o)), "cme_set_solver_opts")


def cme_jacobi_solve(h, n, p0, tol, max_iter, p_out):
    pp, _k0 = _vec_ptr(p0, n)
    po, _k1 = _vec_ptr(p_out, n, writable=True)
    it = C.c_int64()
    st = _lib.cme_jacobi_solve(h, pp, tol, max_iter, po, C.byref(it))
    _chk(st, "cme_jacobi_solve", ok=tuple(SOLVE_STATUS))
    return st, it.value


def cme_transient(h, n, p0, t, eps, p_out):
    pp, _k0 = _vec_ptr(p0, n)
    po, _k1 = _vec_ptr(p_out, n, writable=True)
    k = C.c_int64()
    _chk(_lib.cme_transient(h, pp, t, eps, po, C.byref(k)), "cme_transient")
    return k.value


def cme_get_report(h):
    r = cme_report()
    _chk(_lib.cme_get_report(h, C.byref(r)), "cme_get_report")
    return r


def cme_spmv(h, n, x, y):
    px, _k0 = _vec_ptr(x, n)
    py, _k1 = _vec_ptr(y, n, writable=True)
    _chk(_lib.cme_spmv(h, px, py), "cme_spmv")


def cme_solver_load(h, n, p0=None):
    pp, _k = _vec_ptr(p0, n)
    _chk(_lib.cme_solver_load(h, pp), "cme_solver_load")


def cme_solver_run(h, blocks):
    _chk(_lib.cme_solver_run(h, blocks), "cme_solver_run")


def cme_solver_fetch(h, n, p_out):
    po, _k = _vec_ptr(p_out, n, writable=True)
    _chk(_lib.cme_solver_fetch(h, po), "cme_solver_fetch")


def cme_get_info(h):
    f = cme_info()
    _chk(_lib.cme_get_info(h, C.byref(f)), "cme_get_info")
    return f


def cme_get_permutation(h, n):
    p = np.empty(n, dtype=np.int32)
    _chk(_lib.cme_get_permutation(h, p.ctypes.data_as(i32p)), "cme_get_permutation")
    return p


def cme_export_packed(h):
    v = cme_packed_view()
    _chk(_lib.cme_export_packed(h, C.byref(v)), "cme_export_packed")

    def cp(ptr, k, dt):
        return np.ctypeslib.as_array(ptr, shape=(k,)).astype(dt, copy=True) if k and ptr else np.zeros(0, dt)

    nb = max(1, v.batch)
    out = dict(n=v.n, n_slots=v.n_slots, n_slices=v.n_slices, n_ell=v.n_ell, band_on=bool(v.band_on),
               window=v.window, batch=nb, lo=cp(v.lo, v.n_slots * nb, np.float64),
               up=cp(v.up, v.n_slots * nb, np.float64),
               inv_d=cp(v.inv_d, v.n_slots * nb, np.float64), row_of=cp(v.row_of, v.n_slots, np.int32),
               slice_off=cp(v.slice_off, v.n_slices + 1, np.int64),
               slice_w=cp(v.slice_w, v.n_slices, np.int32), val=cp(v.val, v.n_ell * nb, np.float64),
               col=cp(v.col, v.n_ell, np.int32))
    if v.csr_row_ptr:
        out["csr_row_ptr"] = cp(v.csr_row_ptr, v.n + 1, np.int64)
    return out


def cme_export_compact(h):
    """Host copies of the compact encoding (include/cme.h cme_export_compact)."""
    v = cme_compact_view()
    _chk(_lib.cme_export_compact(h, C.byref(v)), "cme_export_compact")

    def cp(ptr, k, dt):
        return np.ctypeslib.as_array(ptr, shape=(k,)).astype(dt, copy=True) if k and ptr else np.zeros(0, dt)

    out = dict(col16=cp(v.col16, v.n_ell, np.int16), win_shift=v.win_shift)
    if v.batch <= 1:   # (a batch has only the offsets and the tuple index)
        out["val"] = cp(v.val, v.n_ell, np.float64)
    if v.row8:
        out["row8"] = cp(v.row8, v.n_slots, np.uint8)
    if v.lo:
        out["lo"] = cp(v.lo, v.n_slots, np.float64)
        out["up"] = cp(v.up, v.n_slots, np.float64)
    if v.n_dict:
        out["dict"] = cp(v.dict, v.n_dict * max(1, v.batch), np.float64)
        out["vidx"] = cp(v.vidx, v.n_ell, np.uint16)
        if v.loi:
            out["loi"] = cp(v.loi, v.n_slots, np.uint16)
            out["upi"] = cp(v.upi, v.n_slots, np.uint16)
    return out


def cme_period(h, root=0):
    g = C.c_int64()
    _chk(_lib.cme_period(h, root, C.byref(g)), "cme_period")
    return g.value


def cme_export_xw_plan(h, ncw, stages, n_slices):
    """The x-window chunk plan (tiles x 2 int32), ring chunks needed, widest tile."""
    tiles = (n_slices + ncw - 1) // ncw if ncw > 0 else 0   # (the library rejects ncw < 1)
    plan = np.zeros(max(2 * tiles, 2), np.int32)
    need, span = C.c_int64(0), C.c_int64(0)
    _chk(_lib.cme_export_xw_plan(h, ncw, stages, tiles, plan.ctypes.data_as(i32p), C.byref(need), C.byref(span)),
         "cme_export_xw_plan")
    return plan[:2 * tiles].reshape(tiles, 2), need.value, span.value


def cme_comm_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _chk(_lib.cme_comm_unique_id(buf), "cme_comm_unique_id")
    return bytes(buf)


def cme_comm_init(nranks, rank, uid: bytes, device=-1):
    buf = (C.c_uint8 * 128).from_buffer_copy(uid)
    c = vp()
    _chk(_lib.cme_comm_init(nranks, rank, buf, device, C.byref(c)), "cme_comm_init")
    return c


def cme_comm_init_local(devices):
    """In-process peer-memory group: one communicator per entry of `devices`."""
    devs = np.asarray(devices, dtype=np.int32)
    out = (vp * len(devs))()
    _chk(_lib.cme_comm_init_local(len(devs), devs.ctypes.data_as(i32p), out), "cme_comm_init_local")
    return [vp(c) for c in out]


CME_IPC_BLOB_BYTES = 512


def cme_comm_init_ipc(nranks, rank, device=-1):
    """Multi-process peer-memory transport (one process per GPU)."""
    c = vp()
    _chk(_lib.cme_comm_init_ipc(nranks, rank, device, C.byref(c)), "cme_comm_init_ipc")
    return c


def cme_matrix_ipc_export(h) -> bytes:
    buf = (C.c_uint8 * CME_IPC_BLOB_BYTES)()
    _chk(_lib.cme_matrix_ipc_export(h, buf), "cme_matrix_ipc_export")
    return bytes(buf)


def cme_matrix_ipc_attach(h, blobs):
    """blobs: every rank's cme_matrix_ipc_export bytes, in rank order."""
    data = b"".join(blobs)
    if any(len(b) != CME_IPC_BLOB_BYTES for b in blobs):
        raise ValueError("IPC blobs must be CME_IPC_BLOB_BYTES each")
    buf = (C.c_uint8 * len(data)).from_buffer_copy(data)
    _chk(_lib.cme_matrix_ipc_attach(h, buf), "cme_matrix_ipc_attach")


def cme_matrix_plan_partition(h, nranks, rank):
    _chk(_lib.cme_matrix_plan_partition(h, nranks, rank), "cme_matrix_plan_partition")


def cme_matrix_distribute(h, comm):
    _chk(_lib.cme_matrix_distribute(h, comm), "cme_matrix_distribute")


def cme_export_halo(h):
    v = cme_halo_view()
    _chk(_lib.cme_export_halo(h, C.byref(v)), "cme_export_halo")
    cuts = np.ctypeslib.as_array(v.row_begin, shape=(v.nranks + 1,)).copy()
    span = np.ctypeslib.as_array(v.span, shape=(2 * v.nranks,)).copy().reshape(v.nranks, 2)

    def cp(ptr, k):
        return np.ctypeslib.as_array(ptr, shape=(k,)).copy() if k else np.zeros(0, np.int64)
    send = list(zip(cp(v.send_peer, v.n_send).tolist(), cp(v.send_off, v.n_send).tolist(),
                    cp(v.send_cnt, v.n_send).tolist()))
    recv = list(zip(cp(v.recv_peer, v.n_recv).tolist(), cp(v.recv_off, v.n_recv).tolist(),
                    cp(v.recv_cnt, v.n_recv).tolist()))
    return dict(nranks=v.nranks, rank=v.rank, cuts=cuts, span=span, send=send, recv=recv)


def cme_matrix_destroy(h):
    _lib.cme_matrix_destroy(h)


def cme_comm_destroy(c):
    _lib.cme_comm_destroy(c)


def cme_status_string(s):
    return _lib.cme_status_string(s).decode()


def cme_last_error():
    return _lib.cme_last_error().decode(errors="replace")


def cme_abi_version():
    return _lib.cme_abi_version()


def cme_network_enumerate(net):
    """Enumerate a workloads.Network with the library's enumerator -> (states, row, col, rate)."""
    x0, reac, chg, rates, w, cap = net.arrays()
    reac, chg = np.ascontiguousarray(reac), np.ascontiguousarray(chg)
    c = vp()
    _chk(_lib.cme_network_enumerate(net.m, x0.ctypes.data_as(i32p), net.R, reac.ctypes.data_as(i32p),
                                    chg.ctypes.data_as(i32p), rates.ctypes.data_as(f64p),
                                    w.ctypes.data_as(i32p), cap, C.byref(c)), "cme_network_enumerate")
    return _coo_take(c)


def cme_network_enumerate_gpu(net, device=-1):
    """GPU enumerator (lexicographic state order) -> (states, row, col, rate)."""
    x0, reac, chg, rates, w, cap = net.arrays()
    reac, chg = np.ascontiguousarray(reac), np.ascontiguousarray(chg)
    c = vp()
    _chk(_lib.cme_network_enumerate_gpu(net.m, x0.ctypes.data_as(i32p), net.R, reac.ctypes.data_as(i32p),
                                        chg.ctypes.data_as(i32p), rates.ctypes.data_as(f64p),
                                        w.ctypes.data_as(i32p), cap, device, C.byref(c)),
         "cme_network_enumerate_gpu")
    return _coo_take(c)


def _coo_take(c):
    try:
        n, nnz, m = C.c_int64(), C.c_int64(), (C.c_int32 * 1)()
        S, R_, Cc, V = i32p(), i32p(), i32p(), f64p()
        _chk(_lib.cme_coo_get(c, C.byref(n), C.byref(nnz), m, C.byref(S), C.byref(R_), C.byref(Cc),
                              C.byref(V)), "cme_coo_get")

        def cp(ptr, k, dt):
            return np.ctypeslib.as_array(ptr, shape=(k,)).astype(dt, copy=True) if k else np.zeros(0, dt)
        states = cp(S, n.value * m[0], np.int32).reshape(n.value, m[0])
        return states, cp(R_, nnz.value, np.int32), cp(Cc, nnz.value, np.int32), cp(V, nnz.value, np.float64)
    finally:
        _lib.cme_coo_destroy(c)


# ---- convenience object ------------------------------------------------------------------
class Matrix:
    """Owning wrapper: create -> reorder -> pack -> solve (all work in libcme).

    `rate` of shape (nnz,) is one matrix; shape (batch, nnz) is a batched sweep
    (vectors then hold batch * n values, member-major)."""

    def __init__(self, n, row, col, rate, flags=CME_DIAG_FROM_COLSUMS):
        self.n = int(n)
        rate = np.asarray(rate, dtype=np.float64)
        if rate.ndim == 2:
            self.batch = rate.shape[0]
            self.h = cme_matrix_create_coo_batch(self.n, row, col, rate, flags)
        else:
            self.batch = 1
            self.h = cme_matrix_create_coo(self.n, row, col, rate, flags)

    @classmethod
    def from_network(cls, net, gpu=False):
        """gpu=True: the GPU enumerator (lexicographic state order)."""
        states, r, c, v = cme_network_enumerate_gpu(net) if gpu else cme_network_enumerate(net)
        m = cls(len(states), r, c, v)
        m.states = states
        return m

    def reorder(self, method=CME_ORDER_NONE, root=0):
        cme_reorder(self.h, method, root)
        return self

    def set_permutation(self, new_to_old):
        cme_set_permutation(self.h, new_to_old)
        return self

    def pack(self, fmt=CME_FMT_DIAG_SELL, window=256, band=CME_BAND_AUTO, device=-1):
        cme_pack(self.h, fmt, window, band, device)
        return self

    def set_opts(self, **kw):
        cme_set_solver_opts(self.h, **kw)
        return self

    def solve(self, p0=None, tol=1e-12, max_iter=1_000_000, p_out=None):
        if p_out is None:
            p_out = np.empty(self.n * self.batch)
        st, it = cme_jacobi_solve(self.h, self.n * self.batch, p0, tol, max_iter, p_out)
        return p_out, SOLVE_STATUS[st], it

    def spmv(self, x, y=None):
        if y is None:
            y = np.empty(self.n * self.batch)
        cme_spmv(self.h, self.n * self.batch, x, y)
        return y

    def transient(self, t, p0=None, eps=1e-14, p_out=None):
        """p(t) = exp(A t) p0 by uniformization; returns (p, terms)."""
        if p_out is None:
            p_out = np.empty(self.n)
        terms = cme_transient(self.h, self.n, p0, t, eps, p_out)
        return p_out, terms

    def batch_report(self):
        return cme_get_batch_report(self.h, self.batch)

    def info(self):
        return cme_get_info(self.h)

    def report(self):
        return cme_get_report(self.h)

    def permutation(self):
        return cme_get_permutation(self.h, self.n)

    def packed(self):
        return cme_export_packed(self.h)

    def compact(self):
        return cme_export_compact(self.h)

    def close(self):
        if getattr(self, "h", None):
            cme_matrix_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
