"""ctypes binding of libttlg.so (include/ttlg.h).  Argument marshalling only:
every step of the transposition runs in the library's CUDA kernels.  There is
no fallback: if the shared library is missing this module raises."""
from __future__ import annotations

import ctypes
import os

MAX_RANK = 15
_PKG = os.path.dirname(os.path.abspath(__file__))
# TTLG_LIB: development override (A/B builds of the same sources); the
# product loads the in-tree build
LIB_PATH = os.environ.get("TTLG_LIB") or os.path.join(_PKG, "libttlg.so")

F32, F64 = 0, 1
SCHEMA_AUTO, SCHEMA_COPY, SCHEMA_FML, SCHEMA_FMS, SCHEMA_OD, SCHEMA_OA = -1, 0, 1, 2, 3, 4
SCHEMA_NAMES = {0: "COPY", 1: "FML", 2: "FMS", 3: "OD", 4: "OA"}
SCHEMA_IDS = {v: k for k, v in SCHEMA_NAMES.items()}

STATUS = {0: "TTLG_OK", 1: "TTLG_ERR_INVALID_VALUE", 2: "TTLG_ERR_ALIASING",
          3: "TTLG_ERR_DEVICE", 4: "TTLG_ERR_CUDA", 5: "TTLG_ERR_NO_MEMORY",
          6: "TTLG_ERR_INTERNAL", 7: "TTLG_ERR_UNSUPPORTED"}

# every symbol include/ttlg.h declares (checked by tests/test_abi.py)
EXPORTS = ["ttlg_plan", "ttlg_plan_ex", "ttlg_plan_hints_init", "ttlg_execute",
           "ttlg_plan_destroy", "ttlg_transpose", "ttlg_execute_host", "ttlg_predict_time",
           "ttlg_plan_describe", "ttlg_status_string", "ttlg_schema_name", "ttlg_version",
           "ttlg_model_source", "ttlg_plan_candidates", "ttlg_plan_tune", "ttlg_plan_strided",
           "ttlg_ipc_export", "ttlg_ipc_open", "ttlg_ipc_close", "ttlg_execute_batch"]
MAX_BATCH = 16
IPC_HANDLE_BYTES = 64


class TtlgError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        super().__init__(f"{what}: {STATUS.get(code, code)}")


class PlanHints(ctypes.Structure):
    _fields_ = [("schema", ctypes.c_int32), ("in_dim", ctypes.c_int32),
                ("in_block", ctypes.c_int64), ("out_dim", ctypes.c_int32),
                ("out_block", ctypes.c_int64), ("elem_bytes_override", ctypes.c_int32),
                ("threads", ctypes.c_int32), ("grid", ctypes.c_int32),
                ("no_fusion", ctypes.c_int32), ("variant", ctypes.c_int32)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("schema", ctypes.c_int32), ("dtype", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("fused_rank", ctypes.c_int32),
                ("fused_extents", ctypes.c_int64 * MAX_RANK),
                ("fused_perm", ctypes.c_int32 * MAX_RANK),
                ("access_bytes", ctypes.c_int32),
                ("tile_extents", ctypes.c_int64 * MAX_RANK),
                ("in_dim", ctypes.c_int32), ("out_dim", ctypes.c_int32),
                ("in_run", ctypes.c_int64), ("out_run", ctypes.c_int64),
                ("tile_volume", ctypes.c_int64), ("num_tiles", ctypes.c_int64),
                ("grid", ctypes.c_int32), ("threads", ctypes.c_int32),
                ("smem_bytes", ctypes.c_int32), ("bytes", ctypes.c_int64),
                ("predicted_seconds", ctypes.c_double), ("candidates", ctypes.c_int32),
                ("param_bytes", ctypes.c_int32), ("kernel", ctypes.c_int32),
                ("occupancy", ctypes.c_int32), ("num_features", ctypes.c_int32),
                ("features", ctypes.c_double * 12), ("stages", ctypes.c_int32)]

    def to_dict(self) -> dict:
        d = self.fused_rank
        return {
            "schema": SCHEMA_NAMES.get(self.schema, str(self.schema)),
            "dtype": "f64" if self.dtype == F64 else "f32",
            "rank": self.rank, "fused_rank": d,
            "fused_extents": [int(x) for x in self.fused_extents[:d]],
            "fused_perm": [int(x) for x in self.fused_perm[:d]],
            "access_bytes": self.access_bytes,
            "tile_extents": [int(x) for x in self.tile_extents[:d]],
            "in_dim": self.in_dim, "out_dim": self.out_dim,
            "in_run": self.in_run, "out_run": self.out_run,
            "tile_volume": self.tile_volume, "num_tiles": self.num_tiles,
            "grid": self.grid, "threads": self.threads, "smem_bytes": self.smem_bytes,
            "bytes": self.bytes, "predicted_seconds": self.predicted_seconds,
            "candidates": self.candidates, "param_bytes": self.param_bytes,
            "kernel": ["direct", "tile", "pipe", "quad", "deint", "bulkq", "bulkg",
                       "vec", "phase", "blk", "tmap"][self.kernel],
            "occupancy": self.occupancy, "stages": self.stages,
            "features": [float(x) for x in self.features[:self.num_features]],
        }


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() "
                          "(no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    i64p = ctypes.POINTER(ctypes.c_int64)
    i32p = ctypes.POINTER(ctypes.c_int32)
    sig = {
        "ttlg_plan": ([ctypes.POINTER(P), ctypes.c_int, ctypes.c_int, i64p, i32p], ctypes.c_int),
        "ttlg_plan_ex": ([ctypes.POINTER(P), ctypes.c_int, ctypes.c_int, i64p, i32p,
                          ctypes.POINTER(PlanHints)], ctypes.c_int),
        "ttlg_plan_hints_init": ([ctypes.POINTER(PlanHints)], None),
        "ttlg_plan_strided": ([ctypes.POINTER(P), ctypes.c_int, ctypes.c_int, i64p, i32p, i64p,
                               i64p, ctypes.POINTER(PlanHints)], ctypes.c_int),
        "ttlg_ipc_export": ([P, ctypes.c_char_p, i64p], ctypes.c_int),
        "ttlg_ipc_open": ([ctypes.c_char_p, ctypes.c_int64, ctypes.POINTER(P)], ctypes.c_int),
        "ttlg_ipc_close": ([P, ctypes.c_int64], ctypes.c_int),
        "ttlg_execute": ([P, P, P, P], ctypes.c_int),
        "ttlg_execute_batch": ([P, ctypes.c_int32, ctypes.POINTER(P), ctypes.POINTER(P), P],
                               ctypes.c_int),
        "ttlg_plan_destroy": ([P], ctypes.c_int),
        "ttlg_transpose": ([ctypes.c_int, ctypes.c_int, i64p, i32p, P, P, P], ctypes.c_int),
        "ttlg_execute_host": ([P, P, P, P, P, P], ctypes.c_int),
        "ttlg_predict_time": ([ctypes.c_int, ctypes.c_int, i64p, i32p,
                               ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
        "ttlg_plan_describe": ([P, ctypes.POINTER(PlanInfo)], ctypes.c_int),
        "ttlg_status_string": ([ctypes.c_int], ctypes.c_char_p),
        "ttlg_schema_name": ([ctypes.c_int], ctypes.c_char_p),
        "ttlg_version": ([], ctypes.c_int),
        "ttlg_model_source": ([], ctypes.c_char_p),
        "ttlg_plan_tune": ([ctypes.POINTER(P), P, P, P, ctypes.c_int32,
                            ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
        "ttlg_plan_candidates": ([ctypes.c_int, ctypes.c_int, i64p, i32p, ctypes.POINTER(PlanHints),
                                  ctypes.POINTER(PlanInfo), ctypes.c_int32,
                                  ctypes.POINTER(ctypes.c_int32)], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


lib = _load()


def check(code: int, what: str = "ttlg"):
    if code != 0:
        raise TtlgError(code, what)


def arrays(extents, perm):
    d = len(extents)
    if d != len(perm):
        raise ValueError("extents and perm must have the same length")
    return (ctypes.c_int64 * max(d, 1))(*[int(e) for e in extents]), \
        (ctypes.c_int32 * max(d, 1))(*[int(p) for p in perm])
