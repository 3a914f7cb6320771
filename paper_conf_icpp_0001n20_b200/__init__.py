"""graffix-b200: the B200-native hot path of Graffix (Singh & Nasre, ICPP 2020).

Public API (a thin layer over the C ABI in include/graffix.h):

    ctx = Context(device=0)                       # torch caching allocator hooked in
    g = Graph.upload(ctx, row_ptr, col, w)        # CSR, host (numpy) or device (torch)
    info = g.transform(Knobs(coalesce=True))      # §2/§3/§4 transforms
    run = g.run("sssp", source=-1)                # or "pagerank", "scc", "mst", "bc"
    dist = g.download("dist")                     # per original vertex

All compute runs in libgraffix.so's sm_100a kernels; there is no CPU path.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass, fields

import numpy as np

from ._binding import (ALGOS, ALLOC_FN, COLL_FN, GX_COLL_ALLGATHERV, GX_COLL_ALLREDUCE, GX_COLL_REDUCE_SCATTERV,
                       GX_DT_F32, GX_DT_F64, GX_DT_U32, GX_OP_MIN, GX_ASYNC_UPLOAD, GX_CANONICAL, GX_DL_ASYNC, GX_MAP_AUTO, GX_MAP_LB, GX_MAP_PB, GX_MAP_TPV, GX_MAP_VNS, GX_OUT_BC_F64,
                       GX_OUT_DIST_U32, GX_OUT_LABEL_I32, GX_OUT_MST_WEIGHT_U64, GX_OUT_RANK_F64, GX_W_U8,
                       GX_PTRS_DEVICE, GX_PTRS_HOST, GX_VALIDATE, RELEASE_FN, GraffixError, GxExport,
                       GxExportSizes, GxKnobs, GxRunInfo, GxRunOpts, GxTransformInfo, _check, _ptr, lib)

__all__ = ["Context", "Graph", "Knobs", "GraffixError", "lib", "MAPPINGS"]

MAPPINGS = {"auto": GX_MAP_AUTO, "lb": GX_MAP_LB, "tpv": GX_MAP_TPV, "pb": GX_MAP_PB, "vns": GX_MAP_VNS}


@dataclass
class Knobs:
    """Mirror of gx_knobs; all techniques off = exact mode (paper defaults for parameters)."""
    coalesce: bool = False
    chunk_k: int = 16
    replicate_threshold: float = 0.6
    merge_op: int = 0
    smem: bool = False
    cc_threshold: float = 0.5
    added_edge_budget: int = -1
    smem_iters: int = 0
    smem_max_nodes: int = 64
    degree_norm: bool = False
    degsim_threshold: float = 0.3
    degree_target: float = 0.85
    added_weight: str = "sum"          # N3: "sum" | "max" | "mean" (gx_knobs.added_weight_rule)
    sibling_undirected: bool = False   # N3: §3 sibling edges on the undirected CC view

    def to_c(self) -> GxKnobs:
        k = GxKnobs()
        _check(lib().gx_knobs_default(C.byref(k)))
        for f in fields(self):
            v = getattr(self, f.name)
            if f.name == "added_weight":
                k.added_weight_rule = {"sum": 0, "max": 1, "mean": 2}[v]
                continue
            setattr(k, f.name, int(v) if isinstance(v, bool) else v)
        return k


def hosted_collective(rank: int, group=None):
    """The gx_coll_fn of a hosted context (include/graffix.h): a Python callable
    (kind, host_ptr, count, dtype, op, offsets, world, user) -> 0 / 1 that runs
    the collective with torch.distributed on the host buffer, in place.  The
    allgather-v and reduce-scatter-v travel as an allreduce: sum over a buffer
    holding only this rank's slice (exact: one non-zero term per element), min
    over the whole buffer (a superset of the reduce-scatter).  u32 travels as
    int64 (gloo has no unsigned reductions).  Needs no GPU (the library stages
    device data through pinned host memory before calling it)."""
    import torch
    import torch.distributed as dist
    np_dt = {GX_DT_U32: np.uint32, GX_DT_F32: np.float32, GX_DT_F64: np.float64}

    def _coll(kind, buf, count, dtype, op, offsets, nw, user):
        try:
            if count == 0:
                return 0
            a = np.ctypeslib.as_array((C.c_char * (count * np.dtype(np_dt[dtype]).itemsize)).from_address(buf))
            a = a.view(np_dt[dtype])
            t = torch.from_numpy(a.astype(np.int64) if dtype == GX_DT_U32 else a.copy())
            rop = dist.ReduceOp.MIN if op == GX_OP_MIN else dist.ReduceOp.SUM
            if kind == GX_COLL_ALLGATHERV:
                lo, hi = offsets[rank], offsets[rank + 1]
                t[:lo] = 0
                t[hi:] = 0
                rop = dist.ReduceOp.SUM
            dist.all_reduce(t, op=rop, group=group)
            a[:] = t.numpy().astype(np_dt[dtype])
            return 0
        except Exception as e:   # reported as GX_E_NCCL by the library
            import sys
            print(f"graffix hosted exchange failed: {e!r}", file=sys.stderr)
            return 1
    return _coll


class Context:
    """A CUDA device + stream (+ optional NCCL communicator)."""

    def __init__(self, device: int = 0, stream=None, torch_allocator: bool = True, _handle=None):
        self._h = C.c_void_p()
        self._cbs = None
        self.device = device
        if _handle is not None:
            self._h = _handle
        else:
            _check(lib().gx_ctx_create(C.byref(self._h), device, C.c_void_p(stream) if stream else None))
        if torch_allocator:
            self._hook_torch()

    @classmethod
    def distributed(cls, device: int, rank: int, world: int, group=None, stream=None):
        """One context per rank with an NCCL communicator; the NCCL unique id is
        broadcast with torch.distributed (any backend: the id travels as a Python
        object, so an NCCL-only process group works -- ADVICE r1)."""
        import glob
        import os

        import torch
        import torch.distributed as dist
        if not os.environ.get("GX_NCCL_LIB"):
            # torch's bundled NCCL (avoid mixing two libnccl copies)
            cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "nccl", "lib",
                                           "libnccl.so.2"))
            if cands:
                os.environ["GX_NCCL_LIB"] = os.path.realpath(cands[0])
        obj = [None]
        if rank == 0:
            buf = (C.c_uint8 * 128)()
            _check(lib().gx_get_nccl_unique_id(buf))
            obj = [bytes(buf)]
        if dist.get_backend(group) == "nccl":
            torch.cuda.set_device(device)   # broadcast_object_list stages through the current device
        dist.broadcast_object_list(obj, src=0, group=group)
        h = C.c_void_p()
        ub = (C.c_uint8 * 128)(*obj[0])
        _check(lib().gx_ctx_create_dist(C.byref(h), device, C.c_void_p(stream) if stream else None, rank, world, ub))
        return cls(device, _handle=h)

    @classmethod
    def hosted(cls, device: int, rank: int, world: int, group=None, stream=None):
        """One context per rank whose partitioned-path collectives go through
        torch.distributed on HOST buffers (gx_ctx_create_hosted), e.g. a gloo
        group -- so several processes may share one GPU and still run the
        library's real 1-D partitioned code (staging and transport only; every
        sweep, layout and reduction decision stays in libgraffix).  The
        allgather-v and reduce-scatter-v are carried as an allreduce: sum over
        a buffer holding only this rank's slice, min over the whole buffer."""
        _coll = hosted_collective(rank, group)
        cb = COLL_FN(_coll)
        h = C.c_void_p()
        _check(lib().gx_ctx_create_hosted(C.byref(h), device, C.c_void_p(stream) if stream else None, rank, world,
                                          cb, None))
        ctx = cls(device, _handle=h)
        ctx._coll_cb = cb                    # keep the trampoline alive with the context
        return ctx

    def _hook_torch(self):
        try:
            import torch
        except ImportError:
            return
        if not torch.cuda.is_available():
            return
        dev = self.device
        alloc_fn = torch.cuda.caching_allocator_alloc
        free_fn = torch.cuda.caching_allocator_delete

        def _alloc(nbytes, stream, user):
            try:
                return alloc_fn(int(nbytes), dev, stream or 0)
            except Exception:
                return None

        def _release(ptr, nbytes, stream, user):
            try:
                free_fn(ptr)
            except Exception:   # interpreter shutdown: the process is exiting anyway
                pass

        self._cbs = (ALLOC_FN(_alloc), RELEASE_FN(_release))
        _check(lib().gx_set_allocator(self._h, self._cbs[0], self._cbs[1], None))

    @property
    def stream_ptr(self) -> int:
        s = C.c_void_p()
        _check(lib().gx_ctx_stream(self._h, C.byref(s)))
        return s.value or 0

    def sync(self):
        _check(lib().gx_sync(self._h))

    def close(self):
        if self._h:
            lib().gx_ctx_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Graph:
    """A graph uploaded to one context; holds its transform and run results."""

    def __init__(self, ctx: Context, handle):
        self.ctx = ctx
        self._h = handle
        n, m = C.c_int64(), C.c_int64()
        _check(lib().gx_graph_info(self._h, C.byref(n), C.byref(m)))
        self.n, self.m = n.value, m.value
        self.last_run: dict | None = None

    @classmethod
    def upload(cls, ctx: Context, row_ptr, col, w=None, validate: bool = False, canonical: bool = False,
               async_upload: bool = False):
        """Upload a CSR graph.  numpy arrays => host pointers; torch CUDA tensors => device.
        async_upload (GX_ASYNC_UPLOAD, with canonical host arrays): the weights are copied on a
        second stream; the arrays are kept referenced by the Graph until it is closed.
        uint8 weights (numpy uint8 / torch uint8) are uploaded as bytes (GX_W_U8) and widened
        on the device."""
        dev = hasattr(row_ptr, "is_cuda") and row_ptr.is_cuda
        w8 = w is not None and str(getattr(w, "dtype", "")) in ("uint8", "torch.uint8")
        if not dev:
            row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
            col = np.ascontiguousarray(col, dtype=np.int32)
            w = None if w is None else np.ascontiguousarray(w, dtype=np.uint8 if w8 else np.uint32)
        n = int(row_ptr.shape[0]) - 1
        m = int(col.shape[0])
        flags = (GX_PTRS_DEVICE if dev else GX_PTRS_HOST) | (GX_VALIDATE if validate else 0) | \
            (GX_CANONICAL if canonical else 0) | (GX_ASYNC_UPLOAD if async_upload else 0) | (GX_W_U8 if w8 else 0)
        h = C.c_void_p()
        _check(lib().gx_graph_upload_csr(ctx._h, C.byref(h), n, m, _ptr(row_ptr), _ptr(col), _ptr(w), flags))
        G = cls(ctx, h)
        if async_upload:
            G._keep = (row_ptr, col, w)   # read by the copy until a joining call (include/graffix.h)
        return G

    @classmethod
    def host_only(cls, row_ptr, col, w=None, validate: bool = False):
        """Host-only graph (no device): canonicalise + transform + export.
        Runs on a machine without a GPU; run()/download() raise GX_E_STATE."""
        row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int32)
        w = None if w is None else np.ascontiguousarray(w, dtype=np.uint32)
        h = C.c_void_p()
        _check(lib().gx_graph_create_host(C.byref(h), int(row_ptr.shape[0]) - 1, int(col.shape[0]), _ptr(row_ptr),
                                          _ptr(col), _ptr(w), GX_VALIDATE if validate else 0))
        return cls(None, h)

    def transform(self, knobs: Knobs | None = None) -> dict:
        info = GxTransformInfo()
        k = knobs.to_c() if knobs is not None else None
        _check(lib().gx_transform(self._h, C.byref(k) if k is not None else None, C.byref(info)))
        return {f: getattr(info, f) for f, _ in info._fields_}

    def run(self, algo: str = "sssp", source: int = -1, max_iters: int = 0, tol: float = 1e-9,
            mapping: str = "auto", damping: float = 0.85, check_every: int = 8, use_graphs: bool = True,
            bc_sources=None, profile: bool = False, sim_ranks: int = 0, pr_schedule: str = "async",
            merge_every: int = 1) -> dict:
        o = GxRunOpts()
        _check(lib().gx_run_opts_default(C.byref(o)))
        o.algo = ALGOS[algo]
        o.source = int(source)
        o.max_iters = int(max_iters)
        o.mapping = MAPPINGS[mapping]
        o.tol = float(tol)
        o.damping = float(damping)
        o.check_every = int(check_every)
        o.use_graphs = int(bool(use_graphs))
        o.profile = int(bool(profile))
        o.sim_ranks = int(sim_ranks)
        o.pr_schedule = {"jacobi": 0, "async": 1}[pr_schedule]
        o.merge_every = int(merge_every)
        keep = None
        if bc_sources is not None:
            keep = np.ascontiguousarray(bc_sources, dtype=np.int64)
            o.bc_sources = keep.ctypes.data
            o.n_bc_sources = int(keep.shape[0])
        info = GxRunInfo()
        _check(lib().gx_run_ex(self._h, C.byref(o), C.byref(info)))
        self.last_run = {f: getattr(info, f) for f, _ in info._fields_ if f != "pad_"}
        return self.last_run

    _KINDS = {"dist": (GX_OUT_DIST_U32, np.uint32), "rank": (GX_OUT_RANK_F64, np.float64),
              "label": (GX_OUT_LABEL_I32, np.int32), "bc": (GX_OUT_BC_F64, np.float64),
              "mst_weight": (GX_OUT_MST_WEIGHT_U64, np.uint64)}

    def download(self, kind: str, out=None, async_copy: bool = False):
        """Result by original vertex id.  ``out`` may be a numpy array (pinned or
        pageable host memory) or a torch CUDA tensor (device copy).  async_copy
        (GX_DL_ASYNC, host ``out``): complete only after ``ctx.sync()``."""
        k, dt = self._KINDS[kind]
        count = 1 if kind == "mst_weight" else self.n
        dev = out is not None and hasattr(out, "is_cuda") and out.is_cuda
        if out is None:
            out = np.empty(count, dtype=dt)
        flags = (GX_PTRS_DEVICE if dev else GX_PTRS_HOST) | (GX_DL_ASYNC if async_copy else 0)
        _check(lib().gx_download(self._h, k, _ptr(out), count, flags))
        if kind == "mst_weight" and not dev:
            return int(out[0])
        return out

    def export(self) -> dict:
        """Transformed graph (debug / parity path)."""
        s = GxExportSizes()
        _check(lib().gx_export_sizes(self._h, C.byref(s)))
        arr = {
            "row_ptr": np.empty(s.n_slots + 1, np.int64), "col": np.empty(s.m_slots, np.int32),
            "w": np.empty(s.m_slots, np.uint32), "edge_added": np.empty(s.m_slots, np.uint8),
            "slot_to_orig": np.empty(s.n_slots, np.int32), "slot_kind": np.empty(s.n_slots, np.uint8),
            "sched": np.empty(s.sched_len, np.int32), "tile_ptr": np.empty(s.n_tiles + 1, np.int64),
            "tile_members": np.empty(s.tile_members_len, np.int32), "tile_centre": np.empty(s.n_tiles, np.int32),
            "tile_iters": np.empty(s.n_tiles, np.int32),
        }
        e = GxExport(**{k: v.ctypes.data if v.size else None for k, v in arr.items()})
        _check(lib().gx_export_transformed(self._h, C.byref(e)))
        arr["n_slots"] = s.n_slots
        arr["m_slots"] = s.m_slots
        return arr

    def close(self):
        if self._h:
            lib().gx_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
