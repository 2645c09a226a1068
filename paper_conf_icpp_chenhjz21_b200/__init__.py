"""B200-native BGPQ: a linearizable batched-heap priority queue (Chen et al., ICPP'21).

Thin Python binding over the C ABI in ``include/bgpq.h`` (``libbgpq.so``, built from
``csrc/``).  This module only marshals arguments: torch provides device memory and
streams, every step of INSERT / DELETEMIN runs in the sm_100a kernels of the library.
There is no CPU fallback — if the extension is missing or no GPU is present the calls
raise.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_CSRC = os.path.join(_HERE, "csrc")
_INCLUDE = os.path.join(os.path.dirname(_HERE), "include")
LIB_PATH = os.environ.get("BGPQ_LIB") or os.path.join(_HERE, "libbgpq.so")

NVCC_ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = [*NVCC_ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC"]
BUILD_DIR = os.path.join(_HERE, "build")
# one object per (K, values) kernel table + the host-side C ABI (compiled in parallel)
KERNEL_UNITS = [(k, v) for k in (64, 128, 256, 512, 1024, 2048, 4096) for v in (0, 1)]

BGPQ_OK, BGPQ_EINVAL, BGPQ_ENOMEM, BGPQ_EFULL, BGPQ_ECUDA = 0, -1, -2, -3, -4
FLAG_VALUES, FLAG_SERIAL, FLAG_LOCKS = 1, 2, 4
# GPU node-state encoding (bgpq_ops.cuh); the oracle's encoding differs (see to_oracle_states)
ST_EMPTY, ST_AVAIL, ST_TARGET, ST_MARKED = 0, 1, 2, 3
STAT_NAMES = ("ins_ops", "ins_heapify_ops", "ins_levels", "ins_noop", "ins_swap", "ins_merge",
              "del_ops", "del_refill_ops", "del_levels", "del_lr_merge", "del_lr_skip", "marked",
              "keys_out", "root_spins", "del_lr_nomove", "del_cy_swap")
VALID_K = (64, 128, 256, 512, 1024, 2048, 4096)  # K = 4096 keys only (values do not fit 227 KB)


def _sources():
    return [os.path.join(_CSRC, f) for f in sorted(os.listdir(_CSRC))] + \
        [os.path.join(_INCLUDE, f) for f in sorted(os.listdir(_INCLUDE))]


def build(force: bool = False, verbose: bool = False, jobs: int | None = None) -> str:
    """Compile libbgpq.so for sm_100a in-tree (nvcc cross-compiles without a GPU): the kernel
    tables of every (K, values) instantiation and the C ABI as separate objects, compiled in
    parallel, linked with nvcc -shared."""
    newest = max(os.path.getmtime(p) for p in _sources())
    if not (force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < newest):
        return LIB_PATH
    os.makedirs(BUILD_DIR, exist_ok=True)
    units = [([f"-DBGPQ_K={k}", f"-DBGPQ_V={v}"], os.path.join(_CSRC, "bgpq_kernels.cu"),
              os.path.join(BUILD_DIR, f"kern_{k}_{v}.o")) for k, v in KERNEL_UNITS]
    units.append(([], os.path.join(_CSRC, "bgpq_api.cu"), os.path.join(BUILD_DIR, "api.o")))
    units.append(([], os.path.join(_CSRC, "bgpq_testprim.cu"), os.path.join(BUILD_DIR, "testprim.o")))
    units.append(([], os.path.join(_CSRC, "bgpq_apps.cu"), os.path.join(BUILD_DIR, "apps.o")))
    jobs = jobs or max(1, min(len(units), os.cpu_count() or 1))
    pending, running, logs = list(units), [], []
    while pending or running:
        while pending and len(running) < jobs:
            defs, src, obj = pending.pop(0)
            cmd = ["nvcc", *NVCC_FLAGS, *(["-Xptxas", "-v"] if verbose else []), *defs, "-c", src, "-o", obj]
            running.append((subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True), obj))
        p, obj = running.pop(0)
        out, _ = p.communicate()
        logs.append(out)
        if p.returncode != 0:
            for q, _ in running:
                q.kill()
            raise RuntimeError(f"nvcc failed for {obj}:\n" + out[-4000:])
    cmd = ["nvcc", *NVCC_ARCH, "-shared", "-o", LIB_PATH + ".tmp", *(u[2] for u in units)]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc link failed:\n" + r.stderr[-4000:])
    if verbose:
        print("".join(logs))
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH


_lib = None
_vp, _u64 = ctypes.c_void_p, ctypes.c_uint64


def lib():
    """Load libbgpq.so (fails loudly if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build() first")
        L = ctypes.CDLL(LIB_PATH)
        L.bgpq_create_ex.argtypes = [_u64, ctypes.c_uint32, ctypes.c_uint32]
        L.bgpq_create_ex.restype = _vp
        L.bgpq_create.argtypes = [_u64, ctypes.c_uint32]
        L.bgpq_create.restype = _vp
        L.bgpq_destroy.argtypes = [_vp]
        L.bgpq_insert.argtypes = [_vp, _vp, _vp, _u64, _vp]
        L.bgpq_deletemin.argtypes = [_vp, _vp, _vp, _u64, _vp, _vp]
        L.bgpq_size.argtypes = [_vp, ctypes.POINTER(_u64), _vp]
        L.bgpq_insert_host.argtypes = [_vp, _vp, _vp, _u64, _vp]
        L.bgpq_deletemin_host.argtypes = [_vp, _vp, _vp, _u64, ctypes.POINTER(_u64), _vp]
        L.bgpq_run_mixed.argtypes = [_vp, _vp, _vp, _vp, _u64, _vp, _vp, _vp, _vp, _vp, _vp, _vp]
        L.bgpq_dump.argtypes = [_vp, _vp, _vp, _vp, _vp]
        L.bgpq_slots.argtypes = [_vp]
        L.bgpq_slots.restype = _u64
        L.bgpq_stats.argtypes = [_vp, _vp, ctypes.c_int]
        L.bgpq_set_grid.argtypes = [_vp, ctypes.c_int]
        L.bgpq_grid.argtypes = [_vp]
        L.bgpq_launch_count.restype = _u64
        L.bgpq_set_debug.argtypes = [ctypes.c_uint32]
        L.bgpq_timers.argtypes = [_vp, _vp]
        L.bgpq_test_prim.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.c_int] + [_vp] * 7 + \
            [ctypes.c_uint32] + [_vp] * 5
        L.bgpq_strerror.restype = ctypes.c_char_p
        L.bgpq_last_error_msg.restype = ctypes.c_char_p
        _lib = L
    return _lib


# every symbol include/bgpq.h declares
EXPORTS = ("bgpq_create", "bgpq_create_ex", "bgpq_destroy", "bgpq_insert", "bgpq_deletemin",
           "bgpq_size", "bgpq_insert_host", "bgpq_deletemin_host", "bgpq_run_mixed", "bgpq_dump",
           "bgpq_slots", "bgpq_stats", "bgpq_set_grid", "bgpq_grid", "bgpq_launch_count",
           "bgpq_last_error", "bgpq_last_error_msg", "bgpq_strerror", "bgpq_set_debug", "bgpq_timers",
           "bgpq_test_prim", "bgpq_view")
# every symbol include/bgpq_apps.h declares
APP_EXPORTS = ("bgpq_ks_prepare", "bgpq_ks_root", "bgpq_ks_run", "bgpq_astar_init", "bgpq_astar_run")


class BGPQError(RuntimeError):
    pass


def _check(rc):
    if rc != BGPQ_OK:
        msg = lib().bgpq_last_error_msg().decode() if rc == BGPQ_ECUDA else ""
        raise BGPQError(f"bgpq error {rc}: {lib().bgpq_strerror(rc).decode()} {msg}")


def _ptr(t):
    if t is None:
        return None
    return ctypes.c_void_p(t.data_ptr())


_U32_DTYPES = None


def _dev_buf(t, n, name, dtypes=None):
    """Validate a caller tensor before its raw pointer crosses the C ABI: CUDA, contiguous,
    a 4-byte integer dtype (uint32 bit patterns), at least n entries."""
    global _U32_DTYPES
    if t is None:
        return None
    import torch
    if _U32_DTYPES is None:
        _U32_DTYPES = tuple(d for d in (torch.int32, getattr(torch, "uint32", None)) if d is not None)
    ok_dtypes = dtypes or _U32_DTYPES
    if not t.is_cuda:
        raise ValueError(f"{name}: must be a CUDA tensor")
    if t.dtype not in ok_dtypes:
        raise ValueError(f"{name}: dtype {t.dtype} not in {ok_dtypes}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if t.numel() < n:
        raise ValueError(f"{name}: {t.numel()} entries < {n} required")
    return ctypes.c_void_p(t.data_ptr())


def set_debug(bits: int):
    """Process-wide test switches of the library (include/bgpq.h bgpq_set_debug)."""
    _check(lib().bgpq_set_debug(int(bits)))


def _stream(stream):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def launch_count() -> int:
    return int(lib().bgpq_launch_count())


class BGPQ:
    """One batched-heap priority queue on the current CUDA device.

    Keys / values are torch tensors of dtype int32 or uint32 holding uint32 bit patterns
    (keys are ordered as unsigned).  Calls are asynchronous on the current (or given)
    torch stream, exactly like the C calls they forward to."""

    def __init__(self, capacity: int, K: int = 1024, values: bool = True, serial: bool = False,
                 locks: bool = False):
        """serial: one CTA, one operation at a time (layout equals the sequential model);
        default: insert calls as a level pipeline, deletemin calls on a top CTA with walker
        CTAs, mixed calls with per-node locks; locks=True: per-node-lock execution for every
        call."""
        if K not in VALID_K or (K == 4096 and values):
            raise ValueError(f"K must be one of {VALID_K} (4096: keys only)")
        flags = ((FLAG_VALUES if values else 0) | (FLAG_SERIAL if serial else 0)
                 | (FLAG_LOCKS if locks else 0))
        self._h = lib().bgpq_create_ex(int(capacity), int(K), flags)
        if not self._h:
            raise BGPQError(f"bgpq_create failed ({lib().bgpq_last_error()})")
        self.K, self.capacity, self.values, self.serial = int(K), int(capacity), values, serial
        self.locks = locks

    def close(self):
        if getattr(self, "_h", None):
            try:
                lib().bgpq_destroy(self._h)
            except Exception:  # interpreter shutdown
                pass
            self._h = None

    __del__ = close

    # -- hot path -------------------------------------------------------------------------
    def insert(self, keys, vals=None, stream=None):
        """BGPQ_INSERT of keys (device tensor, n entries) in ceil(n/K) batches."""
        n = keys.numel()
        _check(lib().bgpq_insert(self._h, _dev_buf(keys, n, "keys"), _dev_buf(vals, n, "vals"), n,
                                 _stream(stream)))

    def deletemin(self, n, out_keys=None, out_vals=None, d_count=None, stream=None):
        """BGPQ_DELETEMIN of n keys; returns (out_keys, out_vals) device tensors (length n;
        the first min(n, size) entries are valid, ascending)."""
        import torch
        if out_keys is None:
            out_keys = torch.empty(n, dtype=torch.int32, device="cuda")
        if out_vals is None and self.values:
            out_vals = torch.empty(n, dtype=torch.int32, device="cuda")
        import torch
        _check(lib().bgpq_deletemin(self._h, _dev_buf(out_keys, n, "out_keys"), _dev_buf(out_vals, n, "out_vals"),
                                    int(n), _dev_buf(d_count, 1, "d_count", (torch.int64,)), _stream(stream)))
        return out_keys, out_vals

    def size(self, stream=None) -> int:
        out = _u64(0)
        _check(lib().bgpq_size(self._h, ctypes.byref(out), _stream(stream)))
        return int(out.value)

    # -- host-buffer variants (e2e) ---------------------------------------------------------
    def insert_host(self, keys: np.ndarray, vals: np.ndarray | None = None, stream=None):
        if keys.dtype.itemsize != 4 or not keys.flags.c_contiguous:
            raise ValueError("keys: contiguous 4-byte integers required")
        if vals is not None and (vals.dtype.itemsize != 4 or len(vals) < len(keys) or not vals.flags.c_contiguous):
            raise ValueError("vals: contiguous 4-byte integers, len >= len(keys) required")
        _check(lib().bgpq_insert_host(self._h, keys.ctypes.data_as(_vp),
                                      None if vals is None else vals.ctypes.data_as(_vp),
                                      len(keys), _stream(stream)))

    def deletemin_host(self, n, out_keys: np.ndarray, out_vals: np.ndarray | None = None, stream=None):
        if out_keys.dtype.itemsize != 4 or len(out_keys) < n or not out_keys.flags.c_contiguous:
            raise ValueError("out_keys: contiguous 4-byte integers, len >= n required")
        if out_vals is not None and (out_vals.dtype.itemsize != 4 or len(out_vals) < n):
            raise ValueError("out_vals: 4-byte integers, len >= n required")
        cnt = _u64(0)
        _check(lib().bgpq_deletemin_host(self._h, out_keys.ctypes.data_as(_vp),
                                         None if out_vals is None else out_vals.ctypes.data_as(_vp),
                                         int(n), ctypes.byref(cnt), _stream(stream)))
        return int(cnt.value)

    # -- test / bench extensions --------------------------------------------------------------
    def run_mixed(self, op_types, op_sizes, in_off, in_keys, in_vals, out_keys, out_vals, op_count,
                  lin_ticket=None, stream=None):
        _check(lib().bgpq_run_mixed(self._h, _ptr(op_types), _ptr(op_sizes), _ptr(in_off),
                                    op_types.numel(), _ptr(in_keys), _ptr(in_vals), _ptr(out_keys),
                                    _ptr(out_vals), _ptr(op_count), _ptr(lin_ticket), _stream(stream)))

    def slots(self) -> int:
        return int(lib().bgpq_slots(self._h))

    def dump(self):
        """Quiescent heap copy: (node_keys [slots,K], node_vals, meta [slots,4], header dict)."""
        S, K = self.slots(), self.K
        nk = np.empty(S * K, np.uint32)
        nv = np.empty(S * K, np.uint32) if self.values else None
        meta = np.empty(S * 4, np.uint32)
        hdr = np.empty(4, np.uint64)
        _check(lib().bgpq_dump(self._h, nk.ctypes.data_as(_vp),
                               None if nv is None else nv.ctypes.data_as(_vp),
                               meta.ctypes.data_as(_vp), hdr.ctypes.data_as(_vp)))
        h = {"heapSize": int(hdr[0]), "rootSize": int(hdr[1]), "pbSize": int(hdr[2]),
             "err": int(np.int32(np.uint32(hdr[3])))}
        return nk.reshape(S, K), (None if nv is None else nv.reshape(S, K)), meta.reshape(S, 4), h

    def stats(self) -> dict:
        out = np.zeros(len(STAT_NAMES), np.uint64)
        _check(lib().bgpq_stats(self._h, out.ctypes.data_as(_vp), len(STAT_NAMES)))
        return dict(zip(STAT_NAMES, (int(x) for x in out)))

    def timers(self) -> np.ndarray:
        """The 32 cumulative cycle counters of the handle (set_debug(8 | 128); debug aid)."""
        out = np.zeros(32, np.uint64)
        _check(lib().bgpq_timers(self._h, out.ctypes.data_as(_vp)))
        return out

    def set_grid(self, ctas: int):
        _check(lib().bgpq_set_grid(self._h, int(ctas)))

    def grid(self) -> int:
        return int(lib().bgpq_grid(self._h))


def test_prim(variant: int, K: int, zk, wk, na, nb, ma, zv=None, wv=None):
    """Run one hot-path device primitive on a batch of cases (include/bgpq.h bgpq_test_prim).
    zk / wk: [n_cases, K] int32 CUDA tensors; na / nb / ma: [n_cases] int32 CUDA tensors.
    Returns (xk, xv, yk, yv) as [n_cases, 2K] CUDA tensors (xv / yv None without values)."""
    import torch
    n = zk.shape[0]
    values = zv is not None
    xk = torch.zeros((n, 2 * K), dtype=torch.int32, device=zk.device)
    yk = torch.zeros_like(xk)
    xv = torch.zeros_like(xk) if values else None
    yv = torch.zeros_like(xk) if values else None
    _check(lib().bgpq_test_prim(int(variant), int(K), int(values), _ptr(zk), _ptr(zv), _ptr(wk), _ptr(wv),
                                _ptr(na), _ptr(nb), _ptr(ma), int(n), _ptr(xk), _ptr(xv), _ptr(yk), _ptr(yv),
                                _stream(None)))
    return xk, xv, yk, yv


def to_oracle_states(gpu_states: np.ndarray) -> np.ndarray:
    """Map GPU node states to the oracle encoding (AVAIL=0, EMPTY=1, TARGET=2, MARKED=3)."""
    m = np.array([1, 0, 2, 3], np.uint32)
    return m[gpu_states]
