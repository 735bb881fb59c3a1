"""Python surface of the TTLG C ABI (same names as include/ttlg.h).

Raw-pointer functions (`plan`, `execute`, `transpose`, `predict_time`) mirror
the C calls one to one.  `transpose_tensor` is the torch convenience: torch
tensors are row-major (last axis fastest), the library is FVI-first (DESIGN.md
reading R1), so a torch permute(perm_t) of a rank-d tensor is the library call
with extents_c[k] = shape[d-1-k] and perm_c[i] = d-1-perm_t[d-1-i].
PyTorch supplies device memory and streams only; the data movement is the
library's kernels.
"""
from __future__ import annotations

import ctypes
from typing import Optional, Sequence

from . import _ffi
from ._ffi import (F32, F64, SCHEMA_AUTO, SCHEMA_IDS, TtlgError, PlanHints, PlanInfo,
                   arrays, check, lib)


def _dtype_code(dtype) -> int:
    if isinstance(dtype, int):
        return dtype
    s = str(dtype)
    if s in ("f32", "float32", "torch.float32", "fp32"):
        return F32
    if s in ("f64", "float64", "torch.float64", "fp64"):
        return F64
    raise ValueError(f"unsupported dtype {dtype!r} (fp32/fp64)")


def make_hints(schema=None, in_dim=None, in_block=None, out_dim=None, out_block=None,
               access_bytes=None, threads=None, grid=None, no_fusion=False,
               variant=None) -> PlanHints:
    h = PlanHints()
    lib.ttlg_plan_hints_init(ctypes.byref(h))
    if schema is not None:
        h.schema = SCHEMA_IDS[schema] if isinstance(schema, str) else int(schema)
    if in_dim is not None:
        h.in_dim = in_dim
    if in_block is not None:
        h.in_block = in_block
    if out_dim is not None:
        h.out_dim = out_dim
    if out_block is not None:
        h.out_block = out_block
    if access_bytes is not None:
        h.elem_bytes_override = access_bytes
    if threads is not None:
        h.threads = threads
    if grid is not None:
        h.grid = grid
    h.no_fusion = 1 if no_fusion else 0
    if variant is not None:
        h.variant = variant
    return h


class Plan:
    """A ttlg_plan_t (repeated-use mode)."""

    def __init__(self, dtype, extents: Sequence[int], perm: Sequence[int],
                 in_strides: Optional[Sequence[int]] = None,
                 out_strides: Optional[Sequence[int]] = None, **hints):
        self._h = ctypes.c_void_p()
        self.dtype = _dtype_code(dtype)
        self.extents = [int(e) for e in extents]
        self.perm = [int(p) for p in perm]
        self.strided = in_strides is not None or out_strides is not None
        ext, pr = arrays(self.extents, self.perm)
        if self.strided:
            # sub-tensor form (ttlg_plan_strided): strides in elements
            d = len(self.extents)

            def arr(v):
                if v is None:
                    return None
                if len(v) != d:
                    raise ValueError("strides must have one entry per dim")
                return (ctypes.c_int64 * d)(*[int(x) for x in v])
            hh = make_hints(**hints) if hints else None
            check(lib.ttlg_plan_strided(ctypes.byref(self._h), self.dtype, d, ext, pr,
                                        arr(in_strides), arr(out_strides),
                                        ctypes.byref(hh) if hh is not None else None),
                  "ttlg_plan_strided")
        elif hints:
            hh = make_hints(**hints)
            check(lib.ttlg_plan_ex(ctypes.byref(self._h), self.dtype, len(self.extents), ext, pr,
                                   ctypes.byref(hh)), "ttlg_plan_ex")
        else:
            check(lib.ttlg_plan(ctypes.byref(self._h), self.dtype, len(self.extents), ext, pr),
                  "ttlg_plan")

    @property
    def handle(self):
        return self._h

    def describe(self) -> dict:
        info = PlanInfo()
        check(lib.ttlg_plan_describe(self._h, ctypes.byref(info)), "ttlg_plan_describe")
        return info.to_dict()

    def execute(self, A_ptr: int, B_ptr: int, stream: int = 0):
        check(lib.ttlg_execute(self._h, ctypes.c_void_p(A_ptr), ctypes.c_void_p(B_ptr),
                               ctypes.c_void_p(stream)), "ttlg_execute")

    def execute_batch(self, A_ptrs: Sequence[int], B_ptrs: Sequence[int], stream: int = 0):
        """The plan on len(A_ptrs) (A, B) pairs in one launch (ttlg_execute_batch)."""
        n = len(A_ptrs)
        if len(B_ptrs) != n:
            raise ValueError("A_ptrs and B_ptrs must have the same length")
        a = (ctypes.c_void_p * n)(*[ctypes.c_void_p(int(x)) for x in A_ptrs])
        b = (ctypes.c_void_p * n)(*[ctypes.c_void_p(int(x)) for x in B_ptrs])
        check(lib.ttlg_execute_batch(self._h, n, a, b, ctypes.c_void_p(stream)),
              "ttlg_execute_batch")

    def execute_host(self, A_host: int, B_host: int, A_dev: int, B_dev: int, stream: int = 0):
        check(lib.ttlg_execute_host(self._h, ctypes.c_void_p(A_host), ctypes.c_void_p(B_host),
                                    ctypes.c_void_p(A_dev), ctypes.c_void_p(B_dev),
                                    ctypes.c_void_p(stream)), "ttlg_execute_host")

    def tune(self, A_ptr: int, B_ptr: int, stream: int = 0, max_candidates: int = 8) -> float:
        """Measure-mode refinement (ttlg_plan_tune): time the model's short list on
        these buffers and keep the fastest; returns its measured seconds."""
        out = ctypes.c_double()
        check(lib.ttlg_plan_tune(ctypes.byref(self._h), ctypes.c_void_p(A_ptr),
                                 ctypes.c_void_p(B_ptr), ctypes.c_void_p(stream),
                                 max_candidates, ctypes.byref(out)), "ttlg_plan_tune")
        return out.value

    def destroy(self):
        if self._h:
            lib.ttlg_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def plan(dtype, extents, perm, **hints) -> Plan:
    return Plan(dtype, extents, perm, **hints)


def plan_strided(dtype, extents, perm, in_strides=None, out_strides=None, **hints) -> Plan:
    """Sub-tensor transposition (ttlg_plan_strided): element strides per input
    dim (A) and per output dim (B); None = dense."""
    return Plan(dtype, extents, perm, in_strides=in_strides, out_strides=out_strides, **hints)


# ---- peer memory (CUDA IPC) for the fused sharded exchange ------------------------------
def ipc_export(ptr: int):
    """(handle bytes, offset) of the device allocation containing ptr."""
    h = ctypes.create_string_buffer(_ffi.IPC_HANDLE_BYTES)
    off = ctypes.c_int64()
    check(lib.ttlg_ipc_export(ctypes.c_void_p(ptr), h, ctypes.byref(off)), "ttlg_ipc_export")
    return h.raw, off.value


def ipc_open(handle: bytes, offset: int) -> int:
    """Map another process's allocation on the current device; returns the pointer."""
    out = ctypes.c_void_p()
    check(lib.ttlg_ipc_open(handle, int(offset), ctypes.byref(out)), "ttlg_ipc_open")
    return int(out.value)


def ipc_close(ptr: int, offset: int):
    check(lib.ttlg_ipc_close(ctypes.c_void_p(ptr), int(offset)), "ttlg_ipc_close")


def execute(p: Plan, A_ptr: int, B_ptr: int, stream: int = 0):
    p.execute(A_ptr, B_ptr, stream)


def transpose(dtype, extents, perm, A_ptr: int, B_ptr: int, stream: int = 0):
    """Single-use: ttlg_transpose (plan + launch, no cache, no host sync)."""
    ext, pr = arrays(extents, perm)
    check(lib.ttlg_transpose(_dtype_code(dtype), len(extents), ext, pr, ctypes.c_void_p(A_ptr),
                             ctypes.c_void_p(B_ptr), ctypes.c_void_p(stream)), "ttlg_transpose")


def predict_time(dtype, extents, perm) -> float:
    """Performance-model query (§V; L60-63): predicted seconds."""
    ext, pr = arrays(extents, perm)
    out = ctypes.c_double()
    check(lib.ttlg_predict_time(_dtype_code(dtype), len(extents), ext, pr, ctypes.byref(out)),
          "ttlg_predict_time")
    return out.value


def plan_candidates(dtype, extents, perm, max_out: int = 4096, **hints) -> list:
    """Every candidate slice/schema the planner scores (Alg. 3 enumeration) with its
    model features and predicted seconds (for calibration / regret studies)."""
    ext, pr = arrays(extents, perm)
    out = (PlanInfo * max_out)()
    n = ctypes.c_int32()
    hh = make_hints(**hints) if hints else None
    check(lib.ttlg_plan_candidates(_dtype_code(dtype), len(extents), ext, pr,
                                   ctypes.byref(hh) if hh is not None else None, out, max_out,
                                   ctypes.byref(n)), "ttlg_plan_candidates")
    res = []
    for i in range(n.value):
        d = out[i].to_dict()
        d["hints"] = candidate_hints(d)
        res.append(d)
    return res


def candidate_hints(d: dict) -> dict:
    """Hints that reproduce a candidate returned by plan_candidates()."""
    if d["kernel"] == "deint":
        return {"variant": 4}
    if d["kernel"] == "blk":
        return {"variant": 9}
    a, b = d["in_dim"], d["out_dim"]
    h = {"schema": d["schema"] if d["schema"] != "COPY" else "FML", "in_dim": a,
         "in_block": d["tile_extents"][a], "out_dim": b,
         "out_block": d["tile_extents"][d["fused_perm"][b]], "threads": d["threads"]}
    if d["kernel"] != "direct":
        h["variant"] = {"tile": 1, "pipe": 2, "quad": 3, "deint": 4, "bulkq": 5,
                        "bulkg": 6, "vec": 7, "phase": 8, "tmap": 10}[d["kernel"]]
    if d["kernel"] in ("bulkq", "bulkg", "tmap"):
        h["threads"] = d["threads"] - 32   # consumer threads (warp 0 is the producer)
    return h


def model_source() -> str:
    return lib.ttlg_model_source().decode()


# ---- torch conveniences ---------------------------------------------------------------
def torch_to_c(shape: Sequence[int], perm_t: Sequence[int]):
    """Row-major torch (shape, permute order) -> FVI-first (extents, perm)."""
    d = len(shape)
    ext = [int(shape[d - 1 - k]) for k in range(d)]
    perm = [d - 1 - int(perm_t[d - 1 - i]) for i in range(d)]
    return ext, perm


def _dt_of_tensor(x) -> int:
    if x.element_size() == 8:
        return F64
    if x.element_size() == 4:
        return F32
    raise ValueError("tensor elements must be 4 or 8 bytes")


def transpose_tensor(x, perm_t: Sequence[int], out=None, plan_: Optional[Plan] = None):
    """out = x.permute(perm_t) materialised, computed by the library on x's device
    and current stream.  x and out may be strided views (e.g. slices of larger
    tensors): their strides go to ttlg_plan_strided (the innermost non-unit dim
    of each must be unit-stride; otherwise TtlgError UNSUPPORTED -- there is no
    copy fallback).  `out` defaults to a new contiguous tensor."""
    import torch

    if not x.is_cuda:
        raise ValueError("transpose_tensor needs a CUDA tensor (no CPU path)")
    shape_out = [x.shape[p] for p in perm_t]
    if out is None:
        out = torch.empty(shape_out, dtype=x.dtype, device=x.device)
    elif list(out.shape) != shape_out or out.dtype != x.dtype or out.device != x.device:
        raise ValueError("out must have x.permute(perm_t)'s shape, x's dtype and device")
    if x.numel() == 0:
        return out
    ext, perm = torch_to_c(list(x.shape), perm_t)
    d = len(ext)
    stream = torch.cuda.current_stream(x.device).cuda_stream
    with torch.cuda.device(x.device):
        if plan_ is not None:
            # the plan must describe exactly this (dtype, extents, perm) on dense
            # tensors: a mismatched plan would address past the end of out
            if (plan_.dtype != _dt_of_tensor(x) or plan_.extents != ext or plan_.perm != perm
                    or plan_.strided):
                raise ValueError("plan_ does not match x's dtype / shape / perm_t")
            if not (x.is_contiguous() and out.is_contiguous()):
                raise ValueError("plan_ needs contiguous x and out")
            plan_.execute(x.data_ptr(), out.data_ptr(), stream)
        elif x.is_contiguous() and out.is_contiguous():
            transpose(_dt_of_tensor(x), ext, perm, x.data_ptr(), out.data_ptr(), stream)
        else:
            # FVI-first strides: input dim k is torch dim d-1-k, output dim i is
            # out's torch dim d-1-i
            in_strides = [x.stride(d - 1 - k) for k in range(d)]
            out_strides = [out.stride(d - 1 - i) for i in range(d)]
            plan_strided(_dt_of_tensor(x), ext, perm, in_strides, out_strides).execute(
                x.data_ptr(), out.data_ptr(), stream)
    return out
