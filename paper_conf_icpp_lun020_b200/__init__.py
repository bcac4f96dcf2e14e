"""B200-native recursive-block sparse triangular solve (Lu, Niu & Liu, ICPP'20).

Thin Python binding of the C ABI in include/sptrsv.h.  Every step of the solve
runs in the CUDA library ``libsptrsv_b200.so`` (sm_100a); this module only
marshals arguments (pointers, sizes, strides, the current torch stream).
PyTorch is used for device memory and streams, never for the arithmetic.

    import paper_conf_icpp_lun020_b200 as sp
    plan = sp.sptrsv_analyse(row_ptr, col_idx, val)        # CSR (numpy or torch)
    x = sp.sptrsv_solve(plan, b)                           # b: cuda (n,) or (n, k)
    sp.sptrsv_free(plan)
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _capi as C
from ._capi import SptrsvError  # noqa: F401

__all__ = ["Plan", "sptrsv_analyse", "sptrsv_solve", "sptrsv_free", "analyse", "SptrsvError", "version"]


def version() -> str:
    return C.lib().sptrsv_version().decode()


def _ptr(a):
    """Raw address of a numpy array or torch tensor (None -> NULL)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _is_torch(a) -> bool:
    return type(a).__module__.startswith("torch")


def _as_int32(a):
    if _is_torch(a):
        import torch
        return a.to(torch.int32).contiguous()
    return np.ascontiguousarray(a, dtype=np.int32)


def _dtype_code(val) -> int:
    if _is_torch(val):
        import torch
        if val.dtype == torch.float64:
            return C.R64F
        if val.dtype == torch.float32:
            return C.R32F
    else:
        if val.dtype == np.float64:
            return C.R64F
        if val.dtype == np.float32:
            return C.R32F
    raise TypeError("values must be float64 or float32")


def _stream_handle(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream  # torch.cuda.Stream


class Plan:
    """Owns an sptrsv_plan_t (the preprocessed, blocked matrix on the device)."""

    def __init__(self, handle: int, n: int, dtype_code: int, keep=None, device: int = -1):
        self._h = ctypes.c_void_p(handle)
        self.n = n
        self.dtype_code = dtype_code
        self.device = device
        self._keep = keep

    # ---------------------------------------------------------------- solve
    def solve(self, b, x=None, stream=None):
        return sptrsv_solve(self, b, x, stream=stream)

    # -------------------------------------------------------- introspection
    def info(self) -> dict:
        pi = C.PlanInfo()
        C.check(C.lib().sptrsv_plan_info(self._h, ctypes.byref(pi)), "sptrsv_plan_info")
        d = {f: getattr(pi, f) for f, _ in C.PlanInfo._fields_}
        d["variant"] = [k for k, v in C.VARIANTS.items() if v == pi.variant][0]
        d["selector"] = [k for k, v in C.SELECTORS.items() if v == pi.selector][0]
        return d

    def segments(self) -> list[dict]:
        cnt = ctypes.c_int32(0)
        C.check(C.lib().sptrsv_plan_segments(self._h, None, 0, ctypes.byref(cnt)), "sptrsv_plan_segments")
        arr = (C.SegInfo * max(1, cnt.value))()
        C.check(C.lib().sptrsv_plan_segments(self._h, arr, cnt.value, ctypes.byref(cnt)), "sptrsv_plan_segments")
        out = []
        for s in arr[: cnt.value]:
            d = {f: getattr(s, f) for f, _ in C.SegInfo._fields_}
            d["kind"] = "TRI" if s.kind == 0 else "SQ"
            d["kernel"] = C.KERNELS[s.kernel]
            d["format"] = C.FORMATS[s.format]
            d["impl"] = C.IMPLS[s.impl]
            out.append(d)
        return out

    def perm(self) -> np.ndarray:
        a = np.empty(self.n, dtype=np.int32)
        C.check(C.lib().sptrsv_plan_perm(self._h, a.ctypes.data), "sptrsv_plan_perm")
        return a

    def levels(self) -> np.ndarray:
        a = np.empty(self.n, dtype=np.int32)
        C.check(C.lib().sptrsv_plan_levels(self._h, a.ctypes.data), "sptrsv_plan_levels")
        return a

    def seg_array(self, seg: int, which: int) -> np.ndarray:
        cnt = ctypes.c_int64(0)
        C.check(C.lib().sptrsv_plan_seg_array(self._h, seg, which, None, 0, ctypes.byref(cnt)),
                "sptrsv_plan_seg_array")
        a = np.empty(cnt.value, dtype=np.int32)
        C.check(C.lib().sptrsv_plan_seg_array(self._h, seg, which, a.ctypes.data, cnt.value, ctypes.byref(cnt)),
                "sptrsv_plan_seg_array")
        return a

    def matrix(self):
        """(row_ptr int64, col_idx int32, val) of the permuted matrix P L P^T."""
        info = self.info()
        rp = np.empty(self.n + 1, dtype=np.int64)
        ci = np.empty(info["nnz"], dtype=np.int32)
        va = np.empty(info["nnz"], dtype=np.float64 if self.dtype_code == C.R64F else np.float32)
        C.check(C.lib().sptrsv_plan_matrix(self._h, rp.ctypes.data, ci.ctypes.data, va.ctypes.data),
                "sptrsv_plan_matrix")
        return rp, ci, va

    def hash(self) -> int:
        """64-bit digest of the plan (identical on every rank for the same input)."""
        h = ctypes.c_uint64(0)
        C.check(C.lib().sptrsv_plan_hash(self._h, ctypes.byref(h)), "sptrsv_plan_hash")
        return int(h.value)

    def set_profiling(self, on: bool = True) -> None:
        C.check(C.lib().sptrsv_set_profiling(self._h, 1 if on else 0), "sptrsv_set_profiling")

    def seg_times(self) -> np.ndarray:
        """ms of the last solve: [permute-in, seg 0 .. seg nseg-1, permute-out]."""
        cap = len(self.segments()) + 2
        buf = (ctypes.c_float * cap)()
        cnt = ctypes.c_int32(0)
        C.check(C.lib().sptrsv_seg_times(self._h, buf, cap, ctypes.byref(cnt)), "sptrsv_seg_times")
        return np.array(buf[: cnt.value], dtype=np.float64)

    # ------------------------------------------------------------ lifetime
    def free(self) -> None:
        if self._h is not None and self._h.value:
            C.check(C.lib().sptrsv_free(self._h), "sptrsv_free")
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()


# torch's CUDA caching allocator behind the C ABI's dev_alloc / dev_free hooks
# (include/sptrsv.h): the plan's arena and solve workspace are then torch
# memory (visible in torch.cuda.memory_allocated).  alloc_ctx carries the
# device ordinal + 1.  The ctypes thunks live for the whole process.
def _torch_alloc(nbytes, stream, ctx):
    try:
        import torch
        return torch.cuda.caching_allocator_alloc(int(nbytes), device=int(ctx or 1) - 1, stream=int(stream or 0))
    except Exception:  # noqa: BLE001 -- reported to C as NULL -> SPTRSV_ERROR_ALLOC
        return None


def _torch_free(ptr, stream, ctx):
    try:
        import torch
        torch.cuda.caching_allocator_delete(int(ptr))
    except Exception:  # noqa: BLE001 -- interpreter shutdown
        pass


_TORCH_ALLOC = C.DEV_ALLOC(_torch_alloc)
_TORCH_FREE = C.DEV_FREE(_torch_free)


def sptrsv_analyse(row_ptr, col_idx, val, n: int | None = None, fill: str = "L", variant: str = "REC",
                   depth: int = -1, min_block_rows: int = 0, reorder="auto", selector: str = "B200",
                   force_tri_impl: str | None = None, force_sq_impl: str | None = None,
                   host_only: bool = False, sm_count: int = 0, threads: int = 0, stream=None,
                   device: int | None = None, transpose: bool = False, max_nrhs: int = 0,
                   graphs: bool = True, allocator: str | None = "torch", analysis: str = "auto") -> Plan:
    """Preprocess a CSR lower (fill='L') or upper (fill='U') triangular matrix.

    transpose=True: the plan solves A^T x = b for the given A (R31).

    reorder: True = level-set reordering of every triangle (the paper, L231),
    False = none, "auto" = none for supernodal inputs, else level (R29).

    allocator: "torch" = every device allocation of the plan goes through
    torch's CUDA caching allocator (C-ABI dev_alloc hooks); None = cudaMalloc.
    max_nrhs: size the solve workspace now for this many RHS columns.
    graphs: replay repeated solves (same b, x, layout) as one CUDA graph.
    analysis: "auto" = on the GPU when the CSR arrays are CUDA tensors, else on
    the host; "host"; "device" (both give the same plan).
    """
    rp = _as_int32(row_ptr)
    ci = _as_int32(col_idx)
    n = (len(rp) - 1) if n is None else n
    nnz = int(rp[-1]) if n >= 0 and len(rp) else 0
    code = _dtype_code(val)
    if not _is_torch(val):
        val = np.ascontiguousarray(val)
    else:
        val = val.contiguous()
    o = C.Opts()
    C.lib().sptrsv_opts_default(ctypes.byref(o))
    o.variant = C.VARIANTS[variant]
    o.depth = depth
    o.min_block_rows = min_block_rows
    o.reorder = 2 if reorder == "auto" else (0 if reorder else 1)
    o.selector = C.SELECTORS[selector]
    o.force_tri_impl = -1 if force_tri_impl is None else C.IMPLS.index(force_tri_impl)
    o.force_sq_impl = -1 if force_sq_impl is None else C.IMPLS.index(force_sq_impl)
    o.host_only = 1 if host_only else 0
    o.sm_count = sm_count
    o.threads = threads
    o.device = -1
    o.transpose = 1 if transpose else 0
    o.max_nrhs = int(max_nrhs)
    o.graphs = 1 if graphs else 0
    o.analysis = {"auto": 0, "host": 1, "device": 2}[analysis]
    if not host_only:
        import torch
        if torch.cuda.is_available():
            o.device = torch.cuda.current_device() if device is None else int(device)
            if allocator == "torch":
                o.dev_alloc = _TORCH_ALLOC
                o.dev_free = _TORCH_FREE
                o.alloc_ctx = o.device + 1
    h = ctypes.c_void_p()
    st = C.lib().sptrsv_analyse(n, nnz, _ptr(rp), _ptr(ci), _ptr(val), code, C.LOWER if fill == "L" else C.UPPER,
                                ctypes.byref(o), _stream_handle(stream), ctypes.byref(h))
    C.check(st, "sptrsv_analyse")
    return Plan(h.value, n, code, device=o.device)


analyse = sptrsv_analyse


def _layout(t, n):
    """(layout, nrhs, ld) for a 1-D or 2-D (n, k) array/tensor, or None."""
    if t.ndim == 1:
        s = t.stride(0) if _is_torch(t) else t.strides[0] // t.itemsize
        if s == 1:
            return C.COL_MAJOR, 1, max(1, n)
        return C.ROW_MAJOR, 1, s
    if _is_torch(t):
        s0, s1 = t.stride()
    else:
        s0, s1 = (v // t.itemsize for v in t.strides)
    k = t.shape[1]
    if s0 == 1 and s1 >= n:
        return C.COL_MAJOR, k, s1
    if s1 == 1 and s0 >= k:
        return C.ROW_MAJOR, k, s0
    return None


def sptrsv_solve(plan: Plan, b, x=None, stream=None, transposed: bool = False):
    """Solve with b of shape (n,) or (n, k) (any of column-/row-major strides).

    b on the GPU (torch): asynchronous on the given (or current torch) stream.
    b on the host (numpy or CPU torch): copied in, solved, copied back (blocking).
    Returns x (allocated like b when not given).  x may be b (in place).
    transposed=True solves A^T x = b with the same plan (C ABI
    sptrsv_solve_transposed: one RHS, device tensors only).
    """
    n = plan.n
    if b.shape[0] != n:
        raise ValueError(f"b has {b.shape[0]} rows, plan has n={n}")
    # the C ABI carries no dtype: b and x must hold the plan's value type
    # (a float32 x under a float64 plan would be written past its end)
    for name, t in (("b", b), ("x", x)):
        if t is not None and _dtype_code(t) != plan.dtype_code:
            raise TypeError(f"{name} is {t.dtype}, the plan was analysed for "
                            f"{'float64' if plan.dtype_code == C.R64F else 'float32'}")
        if t is not None and _is_torch(t) and t.is_cuda and plan.device >= 0 and t.device.index != plan.device:
            raise ValueError(f"{name} is on cuda:{t.device.index}, the plan on cuda:{plan.device}")
    if _is_torch(b):
        import torch
        if _layout(b, n) is None:
            b = b.contiguous()
        if x is None:
            x = torch.empty_strided(b.shape, b.stride(), dtype=b.dtype, device=b.device)
        if stream is None and b.is_cuda:
            stream = torch.cuda.current_stream(b.device)
    else:
        if _layout(b, n) is None:
            b = np.ascontiguousarray(b)
        if x is None:
            x = np.empty_like(b)
    lb = _layout(b, n)
    lx = _layout(x, n)
    if lx is None or lx[0] != lb[0] or lx[1] != lb[1]:
        raise ValueError("x must have the shape and the layout of b")
    layout, nrhs, ldb = lb
    fn = C.lib().sptrsv_solve_transposed if transposed else C.lib().sptrsv_solve
    st = fn(plan._h, _ptr(b), ldb, _ptr(x), lx[2], nrhs, layout, _stream_handle(stream))
    C.check(st, "sptrsv_solve_transposed" if transposed else "sptrsv_solve")
    return x


def sptrsv_free(plan: Plan) -> None:
    plan.free()
