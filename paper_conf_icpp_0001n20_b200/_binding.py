"""ctypes binding of libgraffix.so (include/graffix.h) -- marshalling only.

Every compute step runs in the library's CUDA kernels; this module converts
numpy / torch arguments to plain pointers and raises GraffixError on a
non-zero gx_status.  There is no CPU fallback: without the built library the
import fails, and without a CUDA device context creation fails.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GX_LIB_PATH") or os.path.join(_HERE, "libgraffix.so")

GX_OK, GX_E_INVALID, GX_E_STATE, GX_E_OOM, GX_E_CUDA, GX_E_NCCL, GX_E_UNSUPPORTED = range(7)
STATUS_NAMES = ["GX_OK", "GX_E_INVALID", "GX_E_STATE", "GX_E_OOM", "GX_E_CUDA", "GX_E_NCCL",
                "GX_E_UNSUPPORTED"]
GX_SSSP, GX_PAGERANK, GX_SCC, GX_MST, GX_BC = 1, 2, 3, 4, 5
ALGOS = {"sssp": GX_SSSP, "pagerank": GX_PAGERANK, "pr": GX_PAGERANK, "scc": GX_SCC, "mst": GX_MST,
         "bc": GX_BC}
GX_MERGE_MEAN, GX_MERGE_MIN = 0, 1
GX_MAP_AUTO, GX_MAP_LB, GX_MAP_TPV, GX_MAP_PB, GX_MAP_VNS = 0, 1, 2, 3, 4
GX_PTRS_HOST, GX_PTRS_DEVICE, GX_VALIDATE, GX_CANONICAL, GX_ASYNC_UPLOAD, GX_DL_ASYNC, GX_W_U8 = 0, 1, 2, 4, 8, 16, 32
GX_OUT_DIST_U32, GX_OUT_RANK_F64, GX_OUT_LABEL_I32, GX_OUT_BC_F64, GX_OUT_MST_WEIGHT_U64 = 1, 2, 3, 4, 5

# every symbol include/graffix.h declares (checked by tests/test_capi_symbols.py)
EXPORTED = [
    "gx_abi_version", "gx_last_error", "gx_ctx_create", "gx_get_nccl_unique_id", "gx_ctx_create_dist",
    "gx_set_allocator", "gx_ctx_destroy", "gx_ctx_stream", "gx_graph_upload_csr", "gx_graph_destroy",
    "gx_graph_info", "gx_knobs_default", "gx_transform", "gx_export_sizes", "gx_export_transformed",
    "gx_run", "gx_run_ex", "gx_run_opts_default", "gx_download", "gx_sync", "gx_graph_create_host",
    "gx_partition_rows", "gx_ctx_create_hosted",
]


class GxKnobs(C.Structure):
    _fields_ = [("struct_size", C.c_uint32), ("coalesce", C.c_int32), ("chunk_k", C.c_int32),
                ("replicate_threshold", C.c_double), ("merge_op", C.c_int32), ("smem", C.c_int32),
                ("cc_threshold", C.c_double), ("added_edge_budget", C.c_int64), ("smem_iters", C.c_int32),
                ("smem_max_nodes", C.c_int32), ("degree_norm", C.c_int32), ("degsim_threshold", C.c_double),
                ("degree_target", C.c_double), ("added_weight_rule", C.c_int32), ("sibling_undirected", C.c_int32)]


class GxTransformInfo(C.Structure):
    _fields_ = [(n, C.c_int64) for n in ("n_slots", "n_holes", "n_replicas", "holes_filled",
                                         "edges_added_coalesce", "edges_added_smem", "edges_added_degnorm",
                                         "n_subgraphs", "subgraph_vertices", "m_slots")] + \
               [("transform_ms", C.c_double), ("extra_space_pct", C.c_double)]


class GxRunInfo(C.Structure):
    _fields_ = [("iterations", C.c_int32), ("converged", C.c_int32), ("loop_ms", C.c_double),
                ("last_delta", C.c_double), ("edges_scanned", C.c_int64), ("bytes_model", C.c_int64),
                ("vertices_active", C.c_int64), ("kernel_launches", C.c_int32), ("sweep_launches", C.c_int32),
                ("sweep_ms", C.c_double), ("sweep_bytes", C.c_int64), ("mapping_used", C.c_int32),
                ("dense_iterations", C.c_int32)]


class GxRunOpts(C.Structure):
    _fields_ = [("struct_size", C.c_uint32), ("algo", C.c_int32), ("source", C.c_int64),
                ("max_iters", C.c_int32), ("mapping", C.c_int32), ("tol", C.c_double), ("damping", C.c_double),
                ("check_every", C.c_int32), ("use_graphs", C.c_int32), ("bc_sources", C.c_void_p),
                ("n_bc_sources", C.c_int64), ("profile", C.c_int32), ("sim_ranks", C.c_int32),
                ("pr_schedule", C.c_int32), ("merge_every", C.c_int32)]


class GxExportSizes(C.Structure):
    _fields_ = [(n, C.c_int64) for n in ("n_slots", "m_slots", "n_tiles", "tile_members_len", "sched_len")]


class GxExport(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in ("row_ptr", "col", "w", "edge_added", "slot_to_orig", "slot_kind",
                                          "sched", "tile_ptr", "tile_members", "tile_centre", "tile_iters")]


ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
RELEASE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
# gx_coll_fn (include/graffix.h, hosted exchange)
COLL_FN = C.CFUNCTYPE(C.c_int, C.c_int32, C.c_void_p, C.c_int64, C.c_int32, C.c_int32, C.POINTER(C.c_int64),
                      C.c_int32, C.c_void_p)
GX_COLL_ALLREDUCE, GX_COLL_ALLGATHERV, GX_COLL_REDUCE_SCATTERV = 0, 1, 2
GX_DT_U32, GX_DT_F32, GX_DT_F64 = 0, 1, 2
GX_OP_SUM, GX_OP_MIN = 0, 1


class GraffixError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


_lib = None


def lib():
    """Load libgraffix.so (in-tree build).  Fails loudly if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_icpp_0001n20_b200.build` "
                          "(or __graft_entry__.build()); there is no CPU fallback")
    L = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
    P, i32, i64, u32, d = C.c_void_p, C.c_int32, C.c_int64, C.c_uint32, C.c_double
    sig = {
        "gx_abi_version": ([], C.c_int),
        "gx_last_error": ([], C.c_char_p),
        "gx_ctx_create": ([C.POINTER(P), C.c_int, P], C.c_int),
        "gx_get_nccl_unique_id": ([P], C.c_int),
        "gx_ctx_create_dist": ([C.POINTER(P), C.c_int, P, C.c_int, C.c_int, P], C.c_int),
        "gx_set_allocator": ([P, ALLOC_FN, RELEASE_FN, P], C.c_int),
        "gx_ctx_destroy": ([P], None),
        "gx_ctx_stream": ([P, C.POINTER(P)], C.c_int),
        "gx_graph_upload_csr": ([P, C.POINTER(P), i64, i64, P, P, P, u32], C.c_int),
        "gx_graph_destroy": ([P], None),
        "gx_graph_info": ([P, C.POINTER(i64), C.POINTER(i64)], C.c_int),
        "gx_knobs_default": ([C.POINTER(GxKnobs)], C.c_int),
        "gx_transform": ([P, C.POINTER(GxKnobs), C.POINTER(GxTransformInfo)], C.c_int),
        "gx_export_sizes": ([P, C.POINTER(GxExportSizes)], C.c_int),
        "gx_export_transformed": ([P, C.POINTER(GxExport)], C.c_int),
        "gx_run": ([P, C.c_int, i64, i32, d, C.POINTER(GxRunInfo)], C.c_int),
        "gx_run_ex": ([P, C.POINTER(GxRunOpts), C.POINTER(GxRunInfo)], C.c_int),
        "gx_run_opts_default": ([C.POINTER(GxRunOpts)], C.c_int),
        "gx_download": ([P, i32, P, i64, u32], C.c_int),
        "gx_sync": ([P], C.c_int),
        "gx_graph_create_host": ([C.POINTER(P), i64, i64, P, P, P, u32], C.c_int),
        "gx_partition_rows": ([i64, P, i32, i64, P], C.c_int),
        "gx_ctx_create_hosted": ([C.POINTER(P), C.c_int, P, C.c_int, C.c_int, COLL_FN, P], C.c_int),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


def _check(st: int):
    if st != GX_OK:
        raise GraffixError(st, lib().gx_last_error().decode(errors="replace"))


def partition_rows(row_ptr, P: int, align: int = 1024):
    """Rank bounds of the 1-D partition (gx_partition_rows)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    out = np.empty(P + 1, dtype=np.int64)
    _check(lib().gx_partition_rows(int(row_ptr.shape[0]) - 1, _ptr(row_ptr), int(P), int(align), _ptr(out)))
    return out


def _ptr(a) -> C.c_void_p:
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        return C.c_void_p(a.data_ptr())
    return C.c_void_p(a.ctypes.data)
