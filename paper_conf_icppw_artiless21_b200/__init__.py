"""Python binding of libturbobc (include/tbc.h): argument marshalling only.

Every step of the TurboBC hot path (Algorithm 1) runs in the CUDA
kernels of ``csrc/``; this module converts numpy / torch arguments to the C ABI and raises
on error.  There is no CPU fallback: if the extension cannot be loaded, import of the
compute entry points raises.

    g = Graph.from_csc(col_ptr, row_idx, directed=False)       # tbc_graph_create_csc
    bc = g.bc(sources)                                          # tbc_bc  -> float64[n]
    depth, sigma = g.bfs(s)                                     # tbc_bfs
    g.bc_device(src_tensor, bc_tensor, stream)                  # tbc_bc_device (accumulates)
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import build as _build

__all__ = ["Graph", "TBCError", "lib", "ENGINE_CSC", "ENGINE_COOT", "DIR_AUTO", "DIR_PUSH", "DIR_PULL",
           "FMT_AUTO", "FMT_LIST", "FMT_STREAM"]

ENGINE_CSC, ENGINE_COOT = 0, 1
FLAG_ONE_FORMAT, FLAG_NO_VALIDATE, FLAG_NO_REORDER = 1, 2, 4
OPT_DIRECTION, OPT_BWD_DIRECTION, OPT_TRACE, OPT_FORMAT, OPT_PARTITIONS = 1, 2, 3, 4, 11
OPT_BATCH, OPT_BATCH_PULL, OPT_BATCH_WIDTH, OPT_BATCH_PARTS, OPT_BATCH_ORDER = 12, 13, 14, 16, 17
OPT_NARROW_WIDTH, OPT_BATCH_LIST, OPT_STAGE, OPT_SIGMA, OPT_NARROW_SLOTS, OPT_BATCH_INPLACE = 18, 19, 20, 21, 22, 23
ENGINE_AUTO, ENGINE_PER_SOURCE, ENGINE_BATCHED, ENGINE_NARROW = -1, 0, 1, 2
OPT_COST = {"list": 5, "stream": 6, "atomic": 7, "vertex": 8, "scan": 9, "bpush": 10}
FMT_AUTO, FMT_LIST, FMT_STREAM = 0, 1, 2
DIR_AUTO, DIR_PUSH, DIR_PULL = 0, 1, 2
STATUS = {0: "TBC_OK", 1: "TBC_ERR_INVALID", 2: "TBC_ERR_OOM", 3: "TBC_ERR_CUDA", 4: "TBC_ERR_UNSUPPORTED"}

# every symbol include/tbc.h declares (checked by tests/test_abi.py)
SYMBOLS = ["tbc_graph_create_csc", "tbc_graph_create_coo", "tbc_bc", "tbc_bc_device", "tbc_bfs",
           "tbc_bfs_batch", "tbc_bfs_batch_ext", "tbc_graph_info", "tbc_graph_set_option", "tbc_stats_get", "tbc_stats_reset", "tbc_trace_get",
           "tbc_profile_get", "tbc_destroy", "tbc_status_string", "tbc_last_error"]


class TBCError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class Stats(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int64) for f in
                ("sources", "reached", "reached_edges", "fwd_edges", "bwd_edges", "levels", "pull_levels", "scans",
                 "max_depth", "list_peak", "bad_sources", "batch_width", "batch_parts", "workspace_bytes",
                 "engine", "list_overflows", "probe_width", "xr_sources")]

    def as_dict(self):
        return {f: int(getattr(self, f)) for f, _ in self._fields_}


_LIB = None


def lib():
    """Load libturbobc.so (building it in-tree first if the sources are newer)."""
    global _LIB
    if _LIB is None:
        path = os.environ.get("TBC_LIB_PATH") or _build.build(debug=os.environ.get("TBC_DEBUG_LIB") == "1",
                                                              variant=os.environ.get("TBC_VARIANT", ""))
        L = ctypes.CDLL(path)
        i64, i32, P = ctypes.c_int64, ctypes.c_int32, ctypes.POINTER
        vp = ctypes.c_void_p
        L.tbc_graph_create_csc.argtypes = [i64, i64, P(i64), P(i32), ctypes.c_int, ctypes.c_int,
                                           ctypes.c_uint, ctypes.c_int, P(vp)]
        L.tbc_graph_create_coo.argtypes = [i64, i64, P(i32), P(i32), ctypes.c_int, ctypes.c_int,
                                           ctypes.c_uint, ctypes.c_int, P(vp)]
        L.tbc_bc.argtypes = [vp, P(i32), i64, P(ctypes.c_double)]
        L.tbc_bc_device.argtypes = [vp, vp, i64, vp, vp]
        L.tbc_bfs.argtypes = [vp, i32, P(i32), P(ctypes.c_double)]
        L.tbc_bfs_batch.argtypes = [vp, P(i32), i64, P(i32), P(ctypes.c_double)]
        L.tbc_bfs_batch_ext.argtypes = [vp, P(i32), i64, P(i32), P(ctypes.c_double), P(i32)]
        L.tbc_graph_info.argtypes = [vp, P(i64), P(i64), P(ctypes.c_int), P(ctypes.c_size_t)]
        L.tbc_graph_set_option.argtypes = [vp, ctypes.c_int, ctypes.c_double]
        L.tbc_stats_get.argtypes = [vp, P(Stats)]
        L.tbc_stats_reset.argtypes = [vp]
        L.tbc_trace_get.argtypes = [vp, P(i64), i64, P(i64)]
        L.tbc_profile_get.argtypes = [vp, P(ctypes.c_uint64), i64, P(i64)]
        L.tbc_destroy.argtypes = [vp]
        L.tbc_status_string.argtypes = [ctypes.c_int]
        L.tbc_status_string.restype = ctypes.c_char_p
        L.tbc_last_error.restype = ctypes.c_char_p
        for name in SYMBOLS[:14]:
            getattr(L, name).restype = ctypes.c_int
        _LIB = L
    return _LIB


def _check(status):
    if status != 0:
        raise TBCError(status, lib().tbc_last_error().decode())


def _p(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


class Graph:
    """A graph resident on one GPU (tbc_graph): CSC of A (+ CSR when directed), workspace."""

    def __init__(self, handle, device):
        self._h = ctypes.c_void_p(handle)
        self.device = device
        n, m, d, b = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int(), ctypes.c_size_t()
        _check(lib().tbc_graph_info(self._h, ctypes.byref(n), ctypes.byref(m), ctypes.byref(d), ctypes.byref(b)))
        self.n, self.nnz, self.directed, self.device_bytes = n.value, m.value, bool(d.value), b.value

    @classmethod
    def from_csc(cls, col_ptr, row_idx, directed: bool, engine: int = ENGINE_CSC, device: int = 0,
                 validate: bool = True, reorder: bool = True, one_format: bool = False):
        """one_format: directed graphs keep the CSC alone (TBC_FLAG_ONE_FORMAT, batched engine only)."""
        cp = np.ascontiguousarray(col_ptr, dtype=np.int64)
        ri = np.ascontiguousarray(row_idx, dtype=np.int32)
        n = cp.size - 1
        h = ctypes.c_void_p()
        flags = ((0 if validate else FLAG_NO_VALIDATE) | (0 if reorder else FLAG_NO_REORDER)
                 | (FLAG_ONE_FORMAT if one_format else 0))
        _check(lib().tbc_graph_create_csc(n, int(cp[-1]) if n >= 0 else 0, _p(cp, ctypes.c_int64),
                                          _p(ri, ctypes.c_int32) if ri.size else None, int(directed),
                                          engine, flags, device, ctypes.byref(h)))
        return cls(h.value, device)

    @classmethod
    def from_coo(cls, n, src, dst, directed: bool, engine: int = ENGINE_CSC, device: int = 0,
                 validate: bool = True, reorder: bool = True, one_format: bool = False):
        s = np.ascontiguousarray(src, dtype=np.int32)
        d = np.ascontiguousarray(dst, dtype=np.int32)
        h = ctypes.c_void_p()
        flags = ((0 if validate else FLAG_NO_VALIDATE) | (0 if reorder else FLAG_NO_REORDER)
                 | (FLAG_ONE_FORMAT if one_format else 0))
        _check(lib().tbc_graph_create_coo(int(n), s.size, _p(s, ctypes.c_int32) if s.size else None,
                                          _p(d, ctypes.c_int32) if d.size else None, int(directed), engine,
                                          flags, device, ctypes.byref(h)))
        return cls(h.value, device)

    # ------------------------------------------------------------------ compute
    def bc(self, sources) -> np.ndarray:
        """tbc_bc: host source list -> host float64[n] (overwritten, synchronous)."""
        src = np.ascontiguousarray(sources, dtype=np.int32)
        out = np.empty(self.n, dtype=np.float64)
        _check(lib().tbc_bc(self._h, _p(src, ctypes.c_int32) if src.size else None, src.size,
                            _p(out, ctypes.c_double)))
        return out

    def bc_device(self, sources, bc, stream=None):
        """tbc_bc_device: torch int32 CUDA tensor of sources, ACCUMULATE into float64 CUDA tensor bc."""
        import torch
        assert sources.dtype == torch.int32 and sources.is_cuda and sources.is_contiguous()
        assert bc.dtype == torch.float64 and bc.is_cuda and bc.numel() == self.n
        if stream is None:
            stream = torch.cuda.current_stream(sources.device)
        _check(lib().tbc_bc_device(self._h, ctypes.c_void_p(sources.data_ptr()), sources.numel(),
                                   ctypes.c_void_p(bc.data_ptr()), ctypes.c_void_p(stream.cuda_stream)))
        return bc

    def bfs(self, source: int):
        """tbc_bfs: (depth int32[n], sigma float64[n]); depth(s)=0, unreachable -1."""
        depth = np.empty(self.n, dtype=np.int32)
        sigma = np.empty(self.n, dtype=np.float64)
        _check(lib().tbc_bfs(self._h, int(source), _p(depth, ctypes.c_int32), _p(sigma, ctypes.c_double)))
        return depth, sigma

    def bfs_batch(self, sources):
        """tbc_bfs_batch: forward stage of the batched engine (the one tbc_bc runs) for a source list;
        returns (depth int32[k, n], sigma float64[k, n]), row i for sources[i]."""
        src = np.ascontiguousarray(sources, dtype=np.int32)
        depth = np.empty((src.size, self.n), dtype=np.int32)
        sigma = np.empty((src.size, self.n), dtype=np.float64)
        _check(lib().tbc_bfs_batch(self._h, _p(src, ctypes.c_int32) if src.size else None, src.size,
                                   _p(depth, ctypes.c_int32), _p(sigma, ctypes.c_double)))
        return depth, sigma

    def bfs_batch_ext(self, sources):
        """tbc_bfs_batch_ext: (depth int32[k, n], sigma mantissa float64[k, n], sigma exponent int32[k, n])."""
        src = np.ascontiguousarray(sources, dtype=np.int32)
        depth = np.empty((src.size, self.n), dtype=np.int32)
        mant = np.empty((src.size, self.n), dtype=np.float64)
        expo = np.empty((src.size, self.n), dtype=np.int32)
        _check(lib().tbc_bfs_batch_ext(self._h, _p(src, ctypes.c_int32) if src.size else None, src.size,
                                       _p(depth, ctypes.c_int32), _p(mant, ctypes.c_double), _p(expo, ctypes.c_int32)))
        return depth, mant, expo

    def set_narrow_slots(self, slots: int):
        """Narrow-level engine: sources run concurrently, one CTA each (TBC_OPT_NARROW_SLOTS, 0 auto)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_NARROW_SLOTS, float(slots)))

    def set_sigma_mode(self, mode: int):
        """Narrow-level engine: 0 fp64 sigma with an extended-range re-run on overflow (default), 1 always
        extended range (TBC_OPT_SIGMA)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_SIGMA, float(mode)))

    def info(self) -> dict:
        """tbc_graph_info now (device_bytes includes the engine workspaces allocated so far)."""
        n, m, d, b = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int(), ctypes.c_size_t()
        _check(lib().tbc_graph_info(self._h, ctypes.byref(n), ctypes.byref(m), ctypes.byref(d), ctypes.byref(b)))
        return {"n": n.value, "nnz": m.value, "directed": bool(d.value), "device_bytes": b.value}

    def set_direction(self, mode: int):
        _check(lib().tbc_graph_set_option(self._h, OPT_DIRECTION, float(mode)))

    def set_bwd_direction(self, mode: int):
        """Backward levels: 0 auto, 1 pull over level L's out-edges only, 2 push from level L+1 when possible."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BWD_DIRECTION, float(mode)))

    def set_batch(self, on: int):
        """bc engine (TBC_OPT_BATCH): -1 auto (default: level-width probe), 0 per source (grid),
        1 batched (W = 32 or 64 sources per sweep), 2 narrow-level (one source per CTA)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH, float(on)))

    def set_batch_list(self, factor: int):
        """Batched engine: level-list entries allocated per vertex (TBC_OPT_BATCH_LIST, 1..64, default 2)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_LIST, float(factor)))

    def set_batch_inplace(self, mode: int):
        """Batched engine: backward overwrites sigma with delta_u in place (TBC_OPT_BATCH_INPLACE: 1 on,
        0 off, -1 auto = in place when the separate delta_u rows would not fit the free memory)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_INPLACE, float(mode)))

    def set_stage(self, stage: int):
        """Measurement: 0 forward + backward (default), 1 forward stage only (TBC_OPT_STAGE; bc untouched)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_STAGE, float(stage)))

    def set_narrow_width(self, width: float):
        """Auto engine: probe vertices per level below which the narrow-level engine runs (TBC_OPT_NARROW_WIDTH)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_NARROW_WIDTH, float(width)))

    def set_batch_width(self, width: int):
        """Batched engine: sources per sweep, 32 or 64, or 0 = auto (TBC_OPT_BATCH_WIDTH; tbc.h states the rule)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_WIDTH, float(width)))

    def set_batch_parts(self, parts: int):
        """Batched engine: SM partitions running batches concurrently (1..8; TBC_OPT_BATCH_PARTS)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_PARTS, float(parts)))

    def set_batch_order(self, grouped: int):
        """Batched engine: 1 group the sources by 2-hop out-volume into batches (default), 0 as given."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_ORDER, float(grouped)))

    def set_batch_pull(self, ratio: float):
        """Batched engine: pull a level when frontier out-edges x ratio > nnz (TBC_OPT_BATCH_PULL)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_BATCH_PULL, float(ratio)))

    def set_partitions(self, parts: int):
        """Number of SM partitions running sources concurrently (1..8; TBC_OPT_PARTITIONS)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_PARTITIONS, float(parts)))

    def set_format(self, mode: int):
        """0 auto, 1 list passes only, 2 edge-stream passes only."""
        _check(lib().tbc_graph_set_option(self._h, OPT_FORMAT, float(mode)))

    def set_cost(self, **costs):
        """Per-item cost model in ps: list=, stream=, atomic=, vertex=, scan=, bpush=."""
        for k, v in costs.items():
            _check(lib().tbc_graph_set_option(self._h, OPT_COST[k], float(v)))

    def set_trace(self, source_index: int):
        """Record the per-level timeline of source_index of the next call(s) (-1 = off)."""
        _check(lib().tbc_graph_set_option(self._h, OPT_TRACE, float(source_index)))

    def trace(self):
        """List of per-level records of the traced source (see tbc_trace_get)."""
        cap = 65536
        buf = np.zeros(8 * cap, dtype=np.int64)
        cnt = ctypes.c_int64()
        _check(lib().tbc_trace_get(self._h, _p(buf, ctypes.c_int64), cap, ctypes.byref(cnt)))
        names = ["init", "scan", "push", "pull_edges", "bwd_edges", "owner"]
        rec = buf[: 8 * cnt.value].reshape(-1, 8)
        out = []
        for i, r in enumerate(rec):
            dt = int(r[0] - rec[i - 1][0]) if i > 0 else 0
            out.append({"kind": names[int(r[1])], "level": int(r[2]), "N": int(r[3]), "E": int(r[4]),
                        "a": int(r[5]), "b": int(r[6]), "dt_us": dt / 1e3})
        return out

    PROFILE_REGIONS = (["barrier"] + [f"{m}_{r}" for m in ("push", "pull", "bwd", "bpush")
                                      for r in ("window", "index", "gather", "tail")]
                       + ["stream_push", "stream_pull", "stream_bwd", "pull_owner", "scan", "bwd_owner", "other"]
                       + ["b_push_slots", "b_push_pairs", "b_pull_slots", "b_pull_pairs", "b_bwd_slots", "b_bwd_pairs",
                          "b_edge_slots", "b_owners"])

    def profile(self) -> dict:
        """Region profile of a -DTBC_PROF library (warp-cycles per region; resets on read)."""
        buf = np.zeros(32, dtype=np.uint64)
        cnt = ctypes.c_int64()
        _check(lib().tbc_profile_get(self._h, buf.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), 32,
                                     ctypes.byref(cnt)))
        return {k: int(v) for k, v in zip(self.PROFILE_REGIONS, buf)}

    def stats(self) -> dict:
        st = Stats()
        _check(lib().tbc_stats_get(self._h, ctypes.byref(st)))
        return st.as_dict()

    def reset_stats(self):
        _check(lib().tbc_stats_reset(self._h))

    def close(self):
        if self._h is not None and self._h.value:
            lib().tbc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
