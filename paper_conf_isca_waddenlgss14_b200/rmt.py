"""Thin ctypes binding over librmt.so (include/rmt.h).

Argument marshalling only: every step of the hot path runs in the CUDA
kernels behind the C ABI.  torch is used for device memory and streams.  There
is no CPU fallback: if librmt.so is missing or no sm_100 device is present,
calls raise.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("RMT_LIB") or os.path.join(_HERE, "librmt.so")  # RMT_LIB: experiment builds only

KERNELS = {
    "blackscholes": 0, "binarysearch": 1, "fwt": 2, "prefixsum": 3, "reduction": 4,
    "transpose": 5, "sobel": 6, "floydwarshall": 7, "dct": 8, "matmul": 9,
    "dwthaar1d": 10, "bitonicsort": 11, "binomialoption": 12,
}
VARIANTS = {"none": 0, "intra_smem": 1, "intra_reg": 2, "inter_group": 3, "inter_cluster": 4, "intra_nolds": 5,
            "dup_kernel": 6}
RMT_VARIANTS = ("intra_smem", "intra_reg", "inter_group", "inter_cluster", "intra_nolds", "dup_kernel")
SITES = {"load": 0, "compute": 1, "smem": 2, "store_val": 3, "store_addr": 4}
ABLATIONS = {"full": 0, "nocomm": 1, "inflate": 2}

F32, U32, U64, U8X4, BF16 = 0, 1, 2, 3, 4
_DT_BYTES = {F32: 4, U32: 4, U64: 8, U8X4: 4, BF16: 2}
# rmt dtype of each buffer per kernel (include/rmt.h schema); None = from tensor
SCHEMA = {
    "blackscholes": (F32, F32, F32),
    "binarysearch": (U32, U32, U32),
    "fwt": (F32, F32),
    "prefixsum": (None, None),  # U32, or F32 with dims[2] bit 1 (include/rmt.h)
    "reduction": (U32, U64),
    "transpose": (None, None),
    "sobel": (U8X4, U8X4),
    "floydwarshall": (U32, U32),
    "dct": (F32, F32),
    "matmul": (BF16, BF16, F32),
    "dwthaar1d": (F32, F32),
    "bitonicsort": (U32, U32),
    "binomialoption": (F32, F32),
}
# optional trailing buffers: the FWT cross-shard stage's partner shard, the
# PrefixSum all-gathered rank totals (include/rmt.h)
SCHEMA_EXTRA = {"fwt": (F32,), "prefixsum": (U64,)}


class RmtError(RuntimeError):
    pass


class _Buf(ctypes.Structure):
    _fields_ = [("ptr", ctypes.c_void_p), ("dtype", ctypes.c_int32), ("numel", ctypes.c_int64)]


class _Bufs(ctypes.Structure):
    _fields_ = [("buf", _Buf * 6), ("nbuf", ctypes.c_int32), ("dims", ctypes.c_int64 * 4)]


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RmtError(f"{LIB_PATH} not built: run __graft_entry__.build() "
                           "(python -c 'import __graft_entry__ as g; g.build()')")
        L = ctypes.CDLL(LIB_PATH)
        P, I64, I32, SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
        L.rmt_launch.argtypes = [I32, I32, ctypes.POINTER(_Bufs), I64, P, P, SZ, P]
        L.rmt_launch.restype = I32
        L.rmt_workspace_size.argtypes = [I32, I32, I64, ctypes.POINTER(ctypes.c_int64)]
        L.rmt_workspace_size.restype = SZ
        L.rmt_run_host.argtypes = [I32, I32, ctypes.POINTER(_Bufs), ctypes.POINTER(_Bufs), I64, P, P, P, SZ, P,
                                   ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
        L.rmt_run_host.restype = I32
        L.rmt_run_host_variants.argtypes = [I32, I32, ctypes.POINTER(I32), ctypes.POINTER(_Bufs),
                                            ctypes.POINTER(_Bufs), I64, P, P, ctypes.POINTER(P),
                                            ctypes.POINTER(SZ), P, ctypes.POINTER(ctypes.c_int64),
                                            ctypes.POINTER(ctypes.c_int64)]
        L.rmt_run_host_variants.restype = I32
        L.rmt_run_host_variants_pipelined.argtypes = [I32, I32, ctypes.POINTER(I32), ctypes.POINTER(_Bufs),
                                                      ctypes.POINTER(_Bufs), I64, P, P, ctypes.POINTER(P),
                                                      ctypes.POINTER(SZ), P, P, P, ctypes.POINTER(ctypes.c_int64),
                                                      ctypes.POINTER(ctypes.c_int64)]
        L.rmt_run_host_variants_pipelined.restype = I32
        L.rmt_inject_fault.argtypes = [I32, I32, I32, I64]
        L.rmt_inject_fault.restype = I32
        L.rmt_clear_faults.restype = I32
        L.rmt_set_ablation.argtypes = [I32]
        L.rmt_set_ablation.restype = I32
        L.rmt_last_launch_count.restype = I32
        L.rmt_strerror.argtypes = [I32]
        L.rmt_strerror.restype = ctypes.c_char_p
        L.rmt_last_error.restype = ctypes.c_char_p
        L.rmt_kernel_name.argtypes = [I32]
        L.rmt_kernel_name.restype = ctypes.c_char_p
        L.rmt_variant_name.argtypes = [I32]
        L.rmt_variant_name.restype = ctypes.c_char_p
        L.rmt_probe_cluster_placement.argtypes = [I64, ctypes.POINTER(ctypes.c_int64)]
        L.rmt_probe_cluster_placement.restype = I32
        L.rmt_workspace_status.argtypes = [I32, P, P]
        L.rmt_workspace_status.restype = I32
        L.rmt_set_stress.argtypes = [I32, I32, I32, ctypes.c_longlong]
        L.rmt_set_stress.restype = I32
        L.rmt_ipc_export.argtypes = [P, P, ctypes.POINTER(ctypes.c_int64)]
        L.rmt_ipc_export.restype = I32
        L.rmt_ipc_open.argtypes = [P, I64, ctypes.POINTER(P)]
        L.rmt_ipc_open.restype = I32
        L.rmt_ipc_close.argtypes = [P, I64]
        L.rmt_ipc_close.restype = I32
        _lib = L
    return _lib


def _check(rc: int, what: str):
    if rc != 0:
        L = lib()
        raise RmtError(f"{what}: {L.rmt_strerror(rc).decode()} ({rc}): {L.rmt_last_error().decode()}")


def _tensor_dtype(t) -> int:
    if t.dtype in (torch.float32,):
        return F32
    if t.dtype in (torch.int32, torch.uint32):
        return U32
    raise RmtError(f"cannot infer rmt dtype for {t.dtype}")


class DevPtr:
    """A raw device pointer of `nbytes` bytes usable as an rmt_launch buffer
    (e.g. a peer rank's buffer opened with ipc_open)."""

    def __init__(self, ptr: int, nbytes: int, offset: int = 0):
        self.ptr, self.nbytes, self.offset = int(ptr), int(nbytes), int(offset)


def ipc_export(t: torch.Tensor):
    """(handle bytes, offset) of the device allocation holding tensor t."""
    h = (ctypes.c_char * 64)()
    off = ctypes.c_int64(0)
    _check(lib().rmt_ipc_export(t.data_ptr(), h, ctypes.byref(off)), "rmt_ipc_export")
    return bytes(h), off.value


def ipc_open(handle: bytes, offset: int, nbytes: int) -> DevPtr:
    p = ctypes.c_void_p(0)
    _check(lib().rmt_ipc_open(ctypes.create_string_buffer(handle, 64), int(offset), ctypes.byref(p)),
           "rmt_ipc_open")
    return DevPtr(p.value, nbytes, offset)


def ipc_close(d: DevPtr):
    _check(lib().rmt_ipc_close(d.ptr, d.offset), "rmt_ipc_close")


def _ptr(t):
    if isinstance(t, DevPtr):
        return t.ptr, t.nbytes
    if isinstance(t, torch.Tensor):
        return t.data_ptr(), t.numel() * t.element_size()
    import numpy as np  # host numpy buffers (rmt_run_host)
    assert isinstance(t, np.ndarray) and t.flags["C_CONTIGUOUS"]
    return t.ctypes.data, t.nbytes


def make_bufs(kernel: str, tensors, dims=()) -> _Bufs:
    schema = SCHEMA[kernel]
    if len(tensors) != len(schema):
        schema = schema + SCHEMA_EXTRA.get(kernel, ())
        if len(tensors) != len(schema):
            raise RmtError(f"{kernel}: expected {len(SCHEMA[kernel])} buffers, got {len(tensors)}")
    b = _Bufs()
    b.nbuf = len(tensors)
    for i, (t, dt) in enumerate(zip(tensors, schema)):
        if dt is None:
            dt = _tensor_dtype(t) if isinstance(t, torch.Tensor) else (F32 if t.dtype.kind == "f" else U32)
        p, nbytes = _ptr(t)
        b.buf[i] = _Buf(p, dt, nbytes // _DT_BYTES[dt])
    for i, d in enumerate(dims):
        b.dims[i] = int(d)
    return b


def workspace_size(kernel: str, variant: str, n: int, dims=()) -> int:
    d = (ctypes.c_int64 * 4)(*([int(x) for x in dims] + [0] * (4 - len(dims))))
    return int(lib().rmt_workspace_size(KERNELS[kernel], VARIANTS[variant], int(n), d))


def make_workspace(kernel: str, variant: str, n: int, dims=(), device="cuda"):
    """Zero-filled device workspace (include/rmt.h: zero once at allocation)."""
    sz = workspace_size(kernel, variant, n, dims)
    return torch.zeros(max(sz, 16), dtype=torch.uint8, device=device)


def launch(kernel: str, variant: str, tensors, n: int, err, dims=(), workspace=None, stream=None) -> int:
    """rmt_launch on the current torch stream.  err: int64 device tensor [1]
    (the library adds mismatch counts).  Returns the number of CUDA kernels
    launched."""
    if stream is None:
        stream = torch.cuda.current_stream().cuda_stream
    b = make_bufs(kernel, tensors, dims)
    ws_ptr, ws_bytes = (workspace.data_ptr(), workspace.numel()) if workspace is not None else (None, 0)
    L = lib()
    _check(L.rmt_launch(KERNELS[kernel], VARIANTS[variant], ctypes.byref(b), int(n), err.data_ptr(),
                        ws_ptr, ws_bytes, stream), f"rmt_launch({kernel},{variant})")
    return L.rmt_last_launch_count()


def run_host(kernel: str, variant: str, host, dev, n: int, err_dev, dims=(), workspace=None, stream=None):
    """rmt_run_host: H2D of inputs, launch, D2H of outputs + error count, sync.
    Returns (err_count, h2d_bytes, d2h_bytes)."""
    if stream is None:
        stream = torch.cuda.current_stream().cuda_stream
    hb = make_bufs(kernel, host, dims)
    db = make_bufs(kernel, dev, dims)
    e = ctypes.c_ulonglong(0)
    h2d = ctypes.c_int64(0)
    d2h = ctypes.c_int64(0)
    ws_ptr, ws_bytes = (workspace.data_ptr(), workspace.numel()) if workspace is not None else (None, 0)
    _check(lib().rmt_run_host(KERNELS[kernel], VARIANTS[variant], ctypes.byref(hb), ctypes.byref(db), int(n),
                              ctypes.byref(e), err_dev.data_ptr(), ws_ptr, ws_bytes, stream,
                              ctypes.byref(h2d), ctypes.byref(d2h)), f"rmt_run_host({kernel},{variant})")
    return e.value, h2d.value, d2h.value


def run_host_variants(kernel: str, variants, host, dev, n: int, err_dev, workspaces, dims=(), stream=None):
    """rmt_run_host_variants: H2D of the inputs once, one launch per variant
    (each with its own device error counter err_dev[v] and workspace), D2H of
    the outputs once and of every error count, sync.  err_dev: int64 device
    tensor [len(variants)].  Returns (error counts, h2d_bytes, d2h_bytes)."""
    if stream is None:
        stream = torch.cuda.current_stream().cuda_stream
    nv = len(variants)
    hb = make_bufs(kernel, host, dims)
    db = make_bufs(kernel, dev, dims)
    vids = (ctypes.c_int * nv)(*[VARIANTS[v] for v in variants])
    errs = (ctypes.c_ulonglong * nv)()
    wsp = (ctypes.c_void_p * nv)(*[w.data_ptr() if w is not None else None for w in workspaces])
    wsb = (ctypes.c_size_t * nv)(*[w.numel() if w is not None else 0 for w in workspaces])
    h2d = ctypes.c_int64(0)
    d2h = ctypes.c_int64(0)
    _check(lib().rmt_run_host_variants(KERNELS[kernel], nv, vids, ctypes.byref(hb), ctypes.byref(db), int(n),
                                       errs, err_dev.data_ptr(), wsp, wsb, stream, ctypes.byref(h2d),
                                       ctypes.byref(d2h)), f"rmt_run_host_variants({kernel})")
    return list(errs), h2d.value, d2h.value


def run_host_variants_pipelined(kernel: str, variants, host, dev, n: int, err_dev, workspaces, err_host,
                                streams, dims=()):
    """rmt_run_host_variants_pipelined: enqueue the inputs on streams[0], the
    launches on streams[1], the outputs and error counts on streams[2]; no
    synchronisation.  err_host: a pinned int64 CPU tensor [len(variants)], valid
    after streams[2] is synchronised (as are the host outputs).  Keep the host
    buffer lists alive until then.  Returns (h2d_bytes, d2h_bytes)."""
    nv = len(variants)
    hb = make_bufs(kernel, host, dims)
    db = make_bufs(kernel, dev, dims)
    vids = (ctypes.c_int * nv)(*[VARIANTS[v] for v in variants])
    wsp = (ctypes.c_void_p * nv)(*[w.data_ptr() if w is not None else None for w in workspaces])
    wsb = (ctypes.c_size_t * nv)(*[w.numel() if w is not None else 0 for w in workspaces])
    h2d = ctypes.c_int64(0)
    d2h = ctypes.c_int64(0)
    _check(lib().rmt_run_host_variants_pipelined(KERNELS[kernel], nv, vids, ctypes.byref(hb), ctypes.byref(db),
                                                 int(n), err_host.data_ptr(), err_dev.data_ptr(), wsp, wsb,
                                                 *[s.cuda_stream for s in streams], ctypes.byref(h2d),
                                                 ctypes.byref(d2h)), f"rmt_run_host_variants_pipelined({kernel})")
    return h2d.value, d2h.value


def inject_fault(replica: int, site, bit: int, elem: int):
    s = SITES[site] if isinstance(site, str) else int(site)
    _check(lib().rmt_inject_fault(int(replica), s, int(bit), int(elem)), "rmt_inject_fault")


def clear_faults():
    _check(lib().rmt_clear_faults(), "rmt_clear_faults")


def set_ablation(mode):
    m = ABLATIONS[mode] if isinstance(mode, str) else int(mode)
    _check(lib().rmt_set_ablation(m), "rmt_set_ablation")


STRESS_TAGS, STRESS_SKEW, STRESS_DROP = 1, 2, 4
EWATCHDOG = -6


def set_stress(depth: int = 0, flags: int = 0, skew_ns: int = 0, watchdog_cycles: int = 0):
    """rmt_set_stress (include/rmt.h): queue depth / tags / skew / dropped producer
    for the inter variants, and the watchdog bound.  All zero = timed configuration."""
    _check(lib().rmt_set_stress(int(depth), int(flags), int(skew_ns), int(watchdog_cycles)), "rmt_set_stress")


def workspace_status(variant: str, workspace, stream=None) -> str | None:
    """rmt_workspace_status: None if the inter-group watchdog flag is clear,
    else its rmt_last_error message (the flag is cleared)."""
    if stream is None:
        stream = torch.cuda.current_stream().cuda_stream
    L = lib()
    rc = L.rmt_workspace_status(VARIANTS[variant], workspace.data_ptr() if workspace is not None else None, stream)
    if rc == 0:
        return None
    if rc != EWATCHDOG:
        _check(rc, "rmt_workspace_status")
    return L.rmt_last_error().decode()


def last_launch_count() -> int:
    return lib().rmt_last_launch_count()


def probe_cluster_placement(pairs: int = 4096) -> int:
    """Pairs (of `pairs` 2-CTA clusters) whose two CTAs shared one SM."""
    out = ctypes.c_int64(-1)
    _check(lib().rmt_probe_cluster_placement(int(pairs), ctypes.byref(out)), "rmt_probe_cluster_placement")
    return out.value
