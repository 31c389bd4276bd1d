"""ctypes mirror of include/stencilfuse.h (kept field-for-field identical)."""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libstencilfuse.so")

SP_F32, SP_F64 = 4, 8
ROLE = {"in": 1, "out": 2, "inout": 3, "temp": 4}


class SpTap(ctypes.Structure):
    _fields_ = [("array", ctypes.c_int32), ("dx", ctypes.c_int32), ("dy", ctypes.c_int32),
                ("dz", ctypes.c_int32)]


class SpTerm(ctypes.Structure):
    _fields_ = [("coef", ctypes.c_double), ("a", SpTap), ("has_b", ctypes.c_int32), ("b", SpTap)]


class SpStmt(ctypes.Structure):
    _fields_ = [("out", ctypes.c_int32), ("n_terms", ctypes.c_int32),
                ("terms", ctypes.POINTER(SpTerm))]


class SpKernel(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("n_stmts", ctypes.c_int32),
                ("stmts", ctypes.POINTER(SpStmt)), ("box", ctypes.POINTER(ctypes.c_int64))]


class SpArrayDesc(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("role", ctypes.c_int)]


class SpGrid(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int64), ("ny", ctypes.c_int64), ("nz_local", ctypes.c_int64),
                ("nz_global", ctypes.c_int64), ("z_offset", ctypes.c_int64),
                ("ghost", ctypes.c_int32 * 3), ("zhalo", ctypes.c_int32), ("dtype", ctypes.c_int)]


class SpStmtRef(ctypes.Structure):
    _fields_ = [("kernel", ctypes.c_int32), ("stmt", ctypes.c_int32)]


class SpLayout(ctypes.Structure):
    _fields_ = [("x_pitch", ctypes.c_int64), ("y_alloc", ctypes.c_int64),
                ("z_alloc", ctypes.c_int64), ("origin_x", ctypes.c_int64),
                ("origin_y", ctypes.c_int64), ("origin_z", ctypes.c_int64),
                ("bytes", ctypes.c_int64)]


class SpTileConfig(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("tile_x", "tile_y", "zchunk", "threads", "prefetch",
                                              "block_x", "block_y", "block_cby", "zqueue", "fastpath",
                                              "frame")]


class SpSearchOptions(ctypes.Structure):
    _fields_ = [("generations", ctypes.c_int32), ("population", ctypes.c_int32),
                ("seed", ctypes.c_uint64), ("objective", ctypes.c_int32),
                ("max_group_kernels", ctypes.c_int32), ("reps", ctypes.c_int32),
                ("c_violation", ctypes.c_double), ("c_sm", ctypes.c_double),
                ("n_configs", ctypes.c_int32), ("configs", ctypes.POINTER(SpTileConfig))]


class SpSearchReport(ctypes.Structure):
    _fields_ = [("cost_us", ctypes.c_double), ("dp_cost_us", ctypes.c_double),
                ("unfused_cost_us", ctypes.c_double), ("groups_evaluated", ctypes.c_int32),
                ("fissioned_kernels", ctypes.c_int32), ("generations_run", ctypes.c_int32)]


class SpEdge(ctypes.Structure):
    _fields_ = [("frm", ctypes.c_int32), ("to", ctypes.c_int32), ("kind", ctypes.c_int32),
                ("array", ctypes.c_int32)]


class SpGroupReport(ctypes.Structure):
    _fields_ = [("n_stmts", ctypes.c_int32), ("n_inputs", ctypes.c_int32),
                ("n_stores", ctypes.c_int32), ("n_smem_stages", ctypes.c_int32),
                ("n_reg_stages", ctypes.c_int32), ("ext", ctypes.c_int32 * 4),
                ("z_below", ctypes.c_int32), ("z_above", ctypes.c_int32),
                ("tile_x", ctypes.c_int32), ("tile_y", ctypes.c_int32),
                ("zchunk", ctypes.c_int32), ("threads", ctypes.c_int32),
                ("grid_ctas", ctypes.c_int32), ("regs_per_thread", ctypes.c_int32),
                ("smem_bytes", ctypes.c_int64), ("bytes_alg", ctypes.c_double),
                ("flops_alg", ctypes.c_double), ("bytes_exec", ctypes.c_double),
                ("flops_exec", ctypes.c_double), ("smem_bytes_pt", ctypes.c_double),
                ("block_x", ctypes.c_int32), ("block_y", ctypes.c_int32),
                ("block_cby", ctypes.c_int32), ("t_model_us", ctypes.c_double),
                ("zqueue", ctypes.c_int32), ("est_regs", ctypes.c_int32),
                ("warmup_steps", ctypes.c_int32), ("prefetch", ctypes.c_int32),
                ("instr_pt", ctypes.c_double)]


# every symbol include/stencilfuse.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "sp_comm_unique_id", "sp_comm_create", "sp_comm_create_loopback", "sp_comm_destroy",
    "sp_signal_buffer", "sp_bind_peer", "sp_bind_peer_signal", "sp_ipc_export", "sp_ipc_open", "stencil_program_create",
    "stencil_program_destroy", "stencil_program_layout", "stencil_program_bind",
    "sp_program_set_option", "sp_program_counts", "sp_program_edges", "sp_fission_components",
    "fusion_plan_set", "sp_plan_greedy", "sp_plan_search", "sp_plan_search_ex", "sp_plan_count", "sp_plan_report", "fusion_plan_report", "sp_plan_source",
    "sp_plan_exchange", "sp_plan_wave_offsets", "sp_plan_tune", "sp_compile", "sp_load", "run_unfused", "run_fused", "sp_run_launch", "sp_run_launch_count", "sp_plan_dag", "exchange_halos", "sp_last_error",
]

_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with __graft_entry__.build() "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        P = ctypes.POINTER
        sig = {
            "sp_comm_unique_id": [vp],
            "sp_comm_create": [vp, i32, i32, P(vp)],
            "sp_comm_create_loopback": [i32, P(vp)],
            "sp_signal_buffer": [vp, P(vp)],
            "sp_bind_peer": [vp, i32, i32, vp],
            "sp_bind_peer_signal": [vp, i32, vp],
            "sp_ipc_export": [vp, vp, P(i64)],
            "sp_ipc_open": [vp, i64, P(vp)],
            "stencil_program_create": [P(SpGrid), i32, P(SpArrayDesc), i32, P(SpKernel), vp, P(vp)],
            "stencil_program_layout": [vp, P(SpLayout)],
            "stencil_program_bind": [vp, i32, vp],
            "sp_program_set_option": [vp, ctypes.c_char_p, i64],
            "sp_program_counts": [vp, P(i32), P(i32)],
            "sp_program_edges": [vp, i32, P(SpEdge), P(i32)],
            "sp_fission_components": [vp, i32, P(i32), P(i32)],
            "fusion_plan_set": [vp, i32, P(i32), P(SpStmtRef)],
            "sp_plan_count": [vp, i32, P(i32)],
            "sp_plan_greedy": [vp, i32, P(i32), P(i32), P(SpStmtRef)],
            "sp_plan_search": [vp, i32, i32, ctypes.c_uint64, i32, P(i32), P(i32), P(SpStmtRef)],
            "sp_plan_search_ex": [vp, P(SpSearchOptions), vp, i32, P(i32), P(i32), P(SpStmtRef),
                                  P(SpTileConfig), P(SpSearchReport)],
            "sp_plan_report": [vp, i32, i32, P(SpGroupReport)],
            "fusion_plan_report": [vp, i32, P(SpGroupReport)],
            "sp_plan_source": [vp, i32, ctypes.c_char_p, ctypes.c_size_t, P(ctypes.c_size_t)],
            "sp_compile": [vp, i32],
            "sp_load": [vp, i32],
            "sp_plan_exchange": [vp, i32, i32, i32, P(i32), P(i32), P(i32), P(i32)],
            "sp_plan_wave_offsets": [vp, i32, P(i32), P(i32)],
            "sp_plan_tune": [vp, i32, i32, P(SpTileConfig)],
            "run_unfused": [vp, vp],
            "run_fused": [vp, vp],
            "sp_run_launch": [vp, i32, i32, vp],
            "sp_run_launch_count": [vp, i32, P(i32)],
            "sp_plan_dag": [vp, i32, i32, i32, P(i32), P(i32), P(i32)],
            "exchange_halos": [vp, i32, P(i32), i32, vp],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.sp_last_error.restype = ctypes.c_char_p
        L.sp_last_error.argtypes = []
        L.stencil_program_destroy.argtypes = [vp]
        L.stencil_program_destroy.restype = None
        L.sp_comm_destroy.argtypes = [vp]
        L.sp_comm_destroy.restype = None
        _lib = L
    return _lib
