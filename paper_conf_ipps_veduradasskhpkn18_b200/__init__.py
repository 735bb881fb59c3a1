"""B200-native TTLG: out-of-place arbitrary-rank tensor transposition for sm_100a.

Public surface (same names as the C ABI in include/ttlg.h):
    plan, execute, transpose, predict_time, Plan, transpose_tensor
plus `sharded` (multi-GPU slab / all-to-all driver over torch.distributed).
"""
from .api import (Plan, plan, execute, transpose, predict_time, transpose_tensor, torch_to_c,
                  make_hints, model_source, plan_candidates, candidate_hints, plan_strided)
from ._ffi import TtlgError, F32, F64, SCHEMA_NAMES, LIB_PATH

__all__ = ["Plan", "plan", "execute", "transpose", "predict_time", "transpose_tensor",
           "torch_to_c", "make_hints", "model_source", "plan_candidates", "candidate_hints", "plan_strided", "TtlgError", "F32", "F64",
           "SCHEMA_NAMES", "LIB_PATH"]
