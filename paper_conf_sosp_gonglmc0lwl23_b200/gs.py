"""Thin Python binding of libgsb200.so (include/gs.h): argument marshalling only.

Every step of the sampling path runs in the library's sm_100a kernels; this
module converts torch tensors to raw pointers, calls the C ABI and wraps the
returned device buffers as torch tensors.  There is no CPU fallback: importing
it without the built library raises.  PyTorch provides the device memory (its
caching allocator is installed as the library's allocator hook) and streams.
"""
from __future__ import annotations

import atexit
import ctypes
import os
import sys

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libgsb200.so")

GS_OK = 0
STATUS = {0: "GS_OK", 1: "GS_ERR_INVALID_ARGUMENT", 2: "GS_ERR_OUT_OF_MEMORY", 3: "GS_ERR_CUDA",
          4: "GS_ERR_UNSORTED_GRAPH", 5: "GS_ERR_INDEX_OUT_OF_RANGE", 6: "GS_ERR_NOT_SUPPORTED",
          7: "GS_ERR_CAPACITY", 8: "GS_ERR_INVALID_GRAPH"}
UNIFORM, EDGE, PASS_COLNORM = 0, 1, 2
LADIES, DEGREE, COUNT = 0, 1, 2
GRAPH_HOST_PTRS, GRAPH_BORROW, GRAPH_HOST_MAPPED = 1, 2, 4
WALK_FORCE_NODE2VEC = 1
META_FIELDS = 8

# Every symbol include/gs.h declares (checked by tests/test_capi_symbols.py).
EXPORTS = ["gs_last_error", "gs_status_string", "gs_version", "gs_kernel_launches", "gs_set_profiling", "gs_blocks_profile",
           "gs_set_allocator",
           "gs_graph_create", "gs_graph_get_info", "gs_graph_destroy", "gs_blocks_sync",
           "gs_blocks_shape", "gs_blocks_view", "gs_blocks_device_meta", "gs_blocks_layer",
           "gs_blocks_pack", "gs_blocks_pack_narrow", "gs_blocks_destroy", "gs_sample_neighbors", "gs_sample_neighbors_ragged",
           "gs_induce_subgraph", "gs_sample_shadow", "gs_sample_saint_rw", "gs_sample_pinsage",
           "gs_sample_layerwise",
           "gs_random_walk", "gs_walk_check", "gs_matrix_slice_columns", "gs_matrix_slice_rows",
           "gs_matrix_sum", "gs_matrix_broadcast", "gs_matrix_elementwise", "gs_matrix_row_ids",
           "gs_matrix_get_view", "gs_matrix_destroy", "gs_matrix_individual_sample",
           "gs_matrix_collective_sample", "gs_matrix_map_reduce", "gs_matrix_asgcn_bias", "gs_pass_attention", "gs_graph_set_weights",
           "gs_graph_cache_hot", "gs_sample_neighbors_hetero", "gs_hetero_block",
           "gs_hetero_frontier", "gs_hetero_destroy"]
OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_POW = 0, 1, 2, 3, 4


class GSError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class _BlockView(ctypes.Structure):
    _fields_ = [("n_cols", ctypes.c_int64), ("n_rows", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("col_map", ctypes.c_void_p), ("row_map", ctypes.c_void_p),
                ("indptr", ctypes.c_void_p), ("row_local", ctypes.c_void_p),
                ("eid", ctypes.c_void_p), ("val", ctypes.c_void_p), ("row_prob", ctypes.c_void_p)]


class _MatrixView(ctypes.Structure):
    _fields_ = [("num_nodes", ctypes.c_int64), ("n_cols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("cols", ctypes.c_void_p), ("indptr", ctypes.c_void_p), ("row", ctypes.c_void_p),
                ("eid", ctypes.c_void_p), ("val", ctypes.c_void_p)]


class _GraphInfo(ctypes.Structure):
    _fields_ = [("num_nodes", ctypes.c_int64), ("num_edges", ctypes.c_int64),
                ("weighted", ctypes.c_int), ("sorted", ctypes.c_int),
                ("max_in_degree", ctypes.c_int64), ("indptr", ctypes.c_void_p),
                ("indices", ctypes.c_void_p), ("weights", ctypes.c_void_p),
                ("host_mapped", ctypes.c_int), ("cached_pages", ctypes.c_int64),
                ("cache_page_entries", ctypes.c_int64)]


class _LayerBuffers(ctypes.Structure):
    _fields_ = [("col_map", ctypes.c_void_p), ("col_capacity", ctypes.c_int64),
                ("row_map", ctypes.c_void_p), ("row_capacity", ctypes.c_int64),
                ("indptr", ctypes.c_void_p), ("indptr_capacity", ctypes.c_int64),
                ("row_local", ctypes.c_void_p), ("eid", ctypes.c_void_p),
                ("val", ctypes.c_void_p), ("edge_capacity", ctypes.c_int64),
                ("row_prob", ctypes.c_void_p)]


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_lib = None
_hooks = None
_exiting = False


@atexit.register
def _at_exit():
    # objects still alive at interpreter exit are leaked on purpose: the CUDA
    # context and PyTorch's allocator may already be torn down.
    global _exiting
    _exiting = True


def _alive():
    return _lib is not None and not _exiting and not sys.is_finalizing()


# Handles released by the garbage collector are destroyed at the next API call
# (never from inside __del__: a GC pass can run while PyTorch's allocator is busy).
_pending = []


def _drain():
    while _pending and _alive():
        kind, h = _pending.pop()
        {"b": _lib.gs_blocks_destroy, "g": _lib.gs_graph_destroy, "m": _lib.gs_matrix_destroy}[kind](h)


def load_library(path: str = LIB_PATH):
    """Loads the C ABI (raises if the CUDA library has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("GS_LIB_PATH", path)  # A/B experiments against another build
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(path)
    vp, i64, i32, u64, u32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_uint32
    L.gs_last_error.restype = ctypes.c_char_p
    L.gs_status_string.restype = ctypes.c_char_p
    L.gs_kernel_launches.restype = ctypes.c_int64
    L.gs_kernel_launches.argtypes = []
    L.gs_set_profiling.argtypes = [ctypes.c_int]
    L.gs_blocks_profile.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(ctypes.c_char_p),
                                    ctypes.POINTER(ctypes.c_double)]
    L.gs_status_string.argtypes = [i32]
    L.gs_set_allocator.argtypes = [_ALLOC_FN, _FREE_FN, vp]
    L.gs_graph_create.argtypes = [vp, vp, vp, i64, i64, u32, vp, ctypes.POINTER(vp)]
    L.gs_graph_get_info.argtypes = [vp, ctypes.POINTER(_GraphInfo)]
    L.gs_graph_destroy.argtypes = [vp]
    L.gs_graph_destroy.restype = None
    L.gs_sample_neighbors.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, i32, u64, vp,
                                      ctypes.POINTER(vp)]
    L.gs_sample_neighbors_ragged.argtypes = [vp, vp, i64, vp, i64, i64, vp, i32, i32, i32, u64, vp,
                                             ctypes.POINTER(vp)]
    L.gs_induce_subgraph.argtypes = [vp, vp, vp, ctypes.POINTER(vp)]
    L.gs_sample_shadow.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, u64, vp, ctypes.POINTER(vp)]
    L.gs_sample_pinsage.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, i32, ctypes.c_float, u64,
                                    vp, ctypes.POINTER(vp)]
    L.gs_pass_attention.argtypes = [vp, vp, i32, vp, vp, i32, vp, vp, vp]
    L.gs_graph_set_weights.argtypes = [vp, vp, ctypes.c_uint32, vp]
    L.gs_graph_cache_hot.argtypes = [vp, i64, vp]
    L.gs_sample_neighbors_hetero.argtypes = [vp, vp, vp, i32, i32, vp, vp, vp, vp, i32, u64, vp,
                                             ctypes.POINTER(vp)]
    L.gs_hetero_block.argtypes = [vp, i32, i32, ctypes.POINTER(vp)]
    L.gs_hetero_frontier.argtypes = [vp, i32, i32, ctypes.POINTER(vp), ctypes.POINTER(ctypes.c_int64)]
    L.gs_hetero_destroy.argtypes = [vp]
    L.gs_hetero_destroy.restype = None
    L.gs_matrix_slice_columns.argtypes = [vp, vp, i64, vp, ctypes.POINTER(vp)]
    L.gs_matrix_slice_rows.argtypes = [vp, vp, i64, vp, ctypes.POINTER(vp)]
    L.gs_matrix_sum.argtypes = [vp, i32, vp, vp]
    L.gs_matrix_individual_sample.argtypes = [vp, i32, i32, i32, u64, i32, i64, vp, ctypes.POINTER(vp)]
    L.gs_matrix_collective_sample.argtypes = [vp, i32, vp, u64, i32, i64, vp, ctypes.POINTER(vp)]
    L.gs_matrix_map_reduce.argtypes = [vp, vp, vp, i32, i32, vp, vp]
    L.gs_matrix_asgcn_bias.argtypes = [vp, vp, i32, vp, vp, vp]
    L.gs_matrix_broadcast.argtypes = [vp, i32, vp, i32, vp]
    L.gs_matrix_elementwise.argtypes = [vp, i32, ctypes.c_float, vp]
    L.gs_matrix_row_ids.argtypes = [vp, vp, ctypes.POINTER(i64), vp]
    L.gs_matrix_get_view.argtypes = [vp, ctypes.POINTER(_MatrixView)]
    L.gs_matrix_destroy.argtypes = [vp]
    L.gs_matrix_destroy.restype = None
    L.gs_sample_saint_rw.argtypes = [vp, vp, i64, i64, i64, i32, u64, vp, ctypes.POINTER(vp)]
    L.gs_sample_layerwise.argtypes = [vp, vp, i64, i64, i64, vp, i32, i32, u64, vp,
                                      ctypes.POINTER(vp)]
    L.gs_random_walk.argtypes = [vp, vp, i64, i64, i32, ctypes.c_float, ctypes.c_float, u64, u32,
                                 vp, vp]
    L.gs_walk_check.argtypes = [vp, vp]
    L.gs_blocks_sync.argtypes = [vp]
    L.gs_blocks_shape.argtypes = [vp, ctypes.POINTER(i64), ctypes.POINTER(i32)]
    L.gs_blocks_view.argtypes = [vp, i64, i32, ctypes.POINTER(_BlockView)]
    L.gs_blocks_device_meta.argtypes = [vp, ctypes.POINTER(vp)]
    L.gs_blocks_layer.argtypes = [vp, i32, ctypes.POINTER(_LayerBuffers)]
    L.gs_blocks_pack.argtypes = [vp, i32, vp, vp, vp, vp, vp, vp]
    L.gs_blocks_pack_narrow.argtypes = [vp, i32, vp, vp, vp, vp, vp, vp]
    L.gs_blocks_destroy.argtypes = [vp]
    L.gs_blocks_destroy.restype = None
    _lib = L
    return L


def _check(st, where=""):
    if st != GS_OK:
        msg = _lib.gs_last_error().decode(errors="replace")
        raise GSError(st, f"{where}: {msg}" if where else msg)


def use_torch_allocator():
    """Routes every library-owned device allocation through PyTorch's caching allocator."""
    global _hooks
    L = load_library()
    if _hooks is not None:  # idempotent: objects keep pointers to these thunks forever
        return

    def _alloc(nbytes, stream, ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), torch.cuda.current_device(),
                                                      stream or 0)
        except Exception:  # reported to C as NULL -> GS_ERR_OUT_OF_MEMORY
            return None

    def _free(ptr, nbytes, stream, ctx):
        torch.cuda.caching_allocator_delete(ptr)

    _hooks = (_ALLOC_FN(_alloc), _FREE_FN(_free))
    _check(L.gs_set_allocator(_hooks[0], _hooks[1], None), "gs_set_allocator")


def _stream_ptr(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


class _CudaArray:
    """__cuda_array_interface__ wrapper so torch can view library-owned memory."""

    def __init__(self, ptr, n, typestr, owner):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr,
                                         "data": (int(ptr or 0), False), "version": 3,
                                         "strides": None}
        self._owner = owner


def _dev_tensor(ptr, n, dtype, owner):
    if n == 0 or not ptr:
        return torch.empty(0, dtype=dtype, device="cuda")
    ts = {torch.int32: "<i4", torch.int64: "<i8", torch.float32: "<f4"}[dtype]
    return torch.as_tensor(_CudaArray(ptr, n, ts, owner), device="cuda")


class Graph:
    """gs_graph: validated CSC in HBM (a0)."""

    def __init__(self, indptr: torch.Tensor, indices: torch.Tensor, weights=None, borrow=False,
                 stream=None, host_mapped=False):
        L = load_library()
        _drain()
        indptr = indptr.to(torch.int64).contiguous()
        indices = indices.to(torch.int32).contiguous()
        if weights is not None:
            weights = weights.to(torch.float32).contiguous()
        flags = 0
        if host_mapped:  # CPU tensors kept in host memory, read over the host link (UVA)
            indptr, indices = indptr.cpu(), indices.cpu()
            weights = None if weights is None else weights.cpu()
            flags |= GRAPH_HOST_PTRS | GRAPH_HOST_MAPPED
            self._keep = (indptr, indices, weights)
        elif indptr.device.type == "cpu":
            flags |= GRAPH_HOST_PTRS
        elif borrow:
            flags |= GRAPH_BORROW
            self._keep = (indptr, indices, weights)
        h = ctypes.c_void_p()
        _check(L.gs_graph_create(_ptr(indptr), _ptr(indices), _ptr(weights), indptr.numel() - 1,
                                 indices.numel(), flags, _stream_ptr(stream), ctypes.byref(h)),
               "gs_graph_create")
        self._h = h
        info = _GraphInfo()
        _check(L.gs_graph_get_info(h, ctypes.byref(info)))
        self.num_nodes = info.num_nodes
        self.num_edges = info.num_edges
        self.weighted = bool(info.weighted)
        self.sorted = bool(info.sorted)
        self.max_in_degree = info.max_in_degree
        self.host_mapped = bool(info.host_mapped)

    @property
    def handle(self):
        return self._h

    def cache_hot(self, budget_bytes: int, stream=None) -> int:
        """Host-mapped graphs: copies the hottest pages of the index / weight
        arrays into HBM (gs_graph_cache_hot, at most budget_bytes); returns the
        number of cached CSC entries."""
        L = load_library()
        _check(L.gs_graph_cache_hot(self._h, ctypes.c_int64(int(budget_bytes)), _stream_ptr(stream)),
               "gs_graph_cache_hot")
        info = _GraphInfo()
        _check(L.gs_graph_get_info(self._h, ctypes.byref(info)))
        return int(info.cached_pages * info.cache_page_entries)

    def set_weights(self, weights: torch.Tensor, borrow: bool = True, stream=None) -> "Graph":
        """Replaces the edge weights (e.g. PASS att) and recomputes the a0 column sums."""
        weights = weights.to(torch.float32).contiguous()
        _check(load_library().gs_graph_set_weights(self._h, _ptr(weights), GRAPH_BORROW if borrow else 0,
                                                   _stream_ptr(stream)), "gs_graph_set_weights")
        self._w = weights
        return self

    def __del__(self):
        try:
            if getattr(self, "_h", None) and _alive():
                _pending.append(("g", self._h))
                self._h = None
        except TypeError:  # interpreter shutdown: module globals already cleared
            pass


class Blocks:
    """gs_blocks: per-(batch, layer) sampled blocks in HBM."""

    def __init__(self):
        self._h = ctypes.c_void_p()
        self.synced = False

    def sync(self):
        _check(_lib.gs_blocks_sync(self._h), "gs_blocks_sync")
        nb, nl = ctypes.c_int64(), ctypes.c_int()
        _check(_lib.gs_blocks_shape(self._h, ctypes.byref(nb), ctypes.byref(nl)))
        self.num_batches, self.num_layers = nb.value, nl.value
        self.synced = True
        return self

    def view(self, batch: int, layer: int) -> dict:
        if not self.synced:
            self.sync()
        v = _BlockView()
        _check(_lib.gs_blocks_view(self._h, batch, layer, ctypes.byref(v)), "gs_blocks_view")
        o = self
        return {
            "col_map": _dev_tensor(v.col_map, v.n_cols, torch.int32, o),
            "row_map": _dev_tensor(v.row_map, v.n_rows, torch.int32, o),
            "indptr": _dev_tensor(v.indptr, v.n_cols + 1, torch.int64, o),
            "row_local": _dev_tensor(v.row_local, v.n_edges, torch.int32, o),
            "eid": _dev_tensor(v.eid, v.n_edges, torch.int64, o),
            "val": None if not v.val else _dev_tensor(v.val, v.n_edges, torch.float32, o),
            "row_prob": None if not v.row_prob else _dev_tensor(v.row_prob, v.n_rows, torch.float32, o),
        }

    def device_meta(self) -> torch.Tensor:
        """int64 [num_batches, num_layers, 8] on the device (no sync)."""
        p = ctypes.c_void_p()
        _check(_lib.gs_blocks_device_meta(self._h, ctypes.byref(p)))
        nb, nl = ctypes.c_int64(), ctypes.c_int()
        _check(_lib.gs_blocks_shape(self._h, ctypes.byref(nb), ctypes.byref(nl)))
        t = _dev_tensor(p.value, nb.value * nl.value * META_FIELDS, torch.int64, self)
        return t.view(nb.value, nl.value, META_FIELDS)

    def layer_capacity(self, layer: int) -> dict:
        """Capacities of layer `layer`'s whole-layer arrays (gs_blocks_layer)."""
        lb = _LayerBuffers()
        _check(_lib.gs_blocks_layer(self._h, layer, ctypes.byref(lb)), "gs_blocks_layer")
        return {"edges": lb.edge_capacity, "indptr": lb.indptr_capacity, "rows": lb.row_capacity}

    def pack(self, layer: int, out: dict = None, stream=None, narrow: bool = False) -> dict:
        """gs_blocks_pack: layer `layer` of every batch packed densely on the
        device (batch order).  Returns device tensors (capacity-sized; the used
        prefix lengths are in `totals` = device int64 [edges, indptr entries, rows]).
        narrow: int32 eid / indptr (gs_blocks_pack_narrow; graphs with < 2^31 entries)."""
        cap = self.layer_capacity(layer)
        wide = torch.int32 if narrow else torch.int64
        if out is not None:  # the C call writes up to the layer's capacity: check the caller's buffers
            for k, n in (("row_local", cap["edges"]), ("eid", cap["edges"]), ("indptr", cap["indptr"]),
                         ("row_map", cap["rows"])):
                if out[k].numel() < n:
                    raise GSError(1, f"pack: out['{k}'] holds {out[k].numel()} < layer capacity {n}")
        if out is None:
            dev = torch.device("cuda", torch.cuda.current_device())
            out = {"row_local": torch.empty(cap["edges"], dtype=torch.int32, device=dev),
                   "eid": torch.empty(cap["edges"], dtype=wide, device=dev),
                   "indptr": torch.empty(cap["indptr"], dtype=wide, device=dev),
                   "row_map": torch.empty(cap["rows"], dtype=torch.int32, device=dev),
                   "totals": torch.empty(3, dtype=torch.int64, device=dev)}
        fn = _lib.gs_blocks_pack_narrow if narrow else _lib.gs_blocks_pack
        for k in ("eid", "indptr"):
            if out[k].dtype != wide:
                raise GSError(1, f"pack: out['{k}'] must be {wide}")
        _check(fn(self._h, layer, _ptr(out["row_local"]), _ptr(out["eid"]), _ptr(out["indptr"]),
                  _ptr(out["row_map"]), _ptr(out["totals"]), _stream_ptr(stream)), "gs_blocks_pack")
        return out

    def to_host(self) -> list:
        """blocks[batch][layer] -> dict of numpy arrays (tests / e2e)."""
        if not self.synced:
            self.sync()
        out = []
        for b in range(self.num_batches):
            layers = []
            for l in range(self.num_layers):
                v = self.view(b, l)
                layers.append({k: (None if x is None else x.cpu().numpy()) for k, x in v.items()})
            out.append(layers)
        return out

    def __del__(self):
        try:
            if getattr(self, "_h", None) and self._h.value and _alive():
                _pending.append(("b", self._h))
                self._h = None
        except TypeError:  # interpreter shutdown: module globals already cleared
            pass


def _host_i32(xs):
    arr = (ctypes.c_int * len(xs))(*[int(x) for x in xs])
    return arr


def sample_neighbors(g: Graph, seeds: torch.Tensor, fanouts, batch_size=None, batch_index_base=0,
                     replace=False, bias_mode=UNIFORM, rng_key=0, stream=None, out: Blocks = None,
                     batch_ptr=None):
    """GraphSAGE / KGCN / weighted A-Res / PASS-style node-wise sampling
    (gs_sample_neighbors; gs_sample_neighbors_ragged when batch_ptr -- a host
    sequence of num_batches + 1 seed offsets -- is given)."""
    L = load_library()
    _drain()
    seeds = seeds.to(torch.int32).contiguous()
    out = out or Blocks()
    f = _host_i32(fanouts)
    if batch_ptr is not None:
        bp = (ctypes.c_int64 * len(batch_ptr))(*[int(x) for x in batch_ptr])
        _check(L.gs_sample_neighbors_ragged(g.handle, _ptr(seeds), seeds.numel(), bp, len(batch_ptr) - 1,
                                            int(batch_index_base), f, len(fanouts), int(replace),
                                            int(bias_mode), ctypes.c_uint64(rng_key), _stream_ptr(stream),
                                            ctypes.byref(out._h)), "gs_sample_neighbors_ragged")
    else:
        bs = int(batch_size or max(1, seeds.numel()))
        _check(L.gs_sample_neighbors(g.handle, _ptr(seeds), seeds.numel(), bs, int(batch_index_base),
                                     f, len(fanouts), int(replace), int(bias_mode),
                                     ctypes.c_uint64(rng_key), _stream_ptr(stream),
                                     ctypes.byref(out._h)), "gs_sample_neighbors")
    out.synced = False
    out._seeds = seeds
    return out


def induce_subgraph(g: Graph, sampled: Blocks, stream=None, out: Blocks = None, retry=True):
    """gs_induce_subgraph: per batch of a node-wise result, the subgraph of A
    induced on its seeds + sampled rows (ascending)."""
    L = load_library()
    _drain()
    out = out or Blocks()
    for attempt in range(3):
        _check(L.gs_induce_subgraph(g.handle, sampled._h, _stream_ptr(stream), ctypes.byref(out._h)),
               "gs_induce_subgraph")
        out.synced = False
        if not retry:
            break
        try:
            out.sync()
            break
        except GSError as e:
            if e.status != 7 or attempt == 2:
                raise
    out._sampled = sampled
    return out


def sample_shadow(g: Graph, seeds: torch.Tensor, fanouts, batch_size=None, batch_index_base=0,
                  bias_mode=UNIFORM, rng_key=0, stream=None, out: Blocks = None, retry=True):
    L = load_library()
    _drain()
    seeds = seeds.to(torch.int32).contiguous()
    bs = int(batch_size or max(1, seeds.numel()))
    out = out or Blocks()
    f = _host_i32(fanouts)
    for attempt in range(3):
        _check(L.gs_sample_shadow(g.handle, _ptr(seeds), seeds.numel(), bs, int(batch_index_base),
                                  f, len(fanouts), int(bias_mode), ctypes.c_uint64(rng_key),
                                  _stream_ptr(stream), ctypes.byref(out._h)), "gs_sample_shadow")
        out.synced = False
        if not retry:
            break
        try:
            out.sync()
            break
        except GSError as e:
            if e.status != 7 or attempt == 2:
                raise
    out._seeds = seeds
    return out


def pass_attention(g: "Graph", X: torch.Tensor, W1: torch.Tensor, W2: torch.Tensor, W3,
                   stream=None, out: torch.Tensor = None) -> torch.Tensor:
    """PASS learned bias att[e] for every edge (Fig. 3(c) lines 3-9; DESIGN R29)
    through gs_pass_attention.  X [N, F], W1/W2 [F, H] bf16 on the device."""
    L = load_library()
    X = X.to(torch.bfloat16).contiguous()
    W1 = W1.to(torch.bfloat16).contiguous()
    W2 = W2.to(torch.bfloat16).contiguous()
    nnz = g.num_edges
    if out is None:
        out = torch.empty(nnz, dtype=torch.float32, device=X.device)
    w3 = (ctypes.c_float * 3)(*[float(x) for x in W3])
    _check(L.gs_pass_attention(g.handle, _ptr(X), X.shape[1], _ptr(W1), _ptr(W2), W1.shape[1], w3,
                               _stream_ptr(stream), _ptr(out)), "gs_pass_attention")
    return out


class Matrix:
    """A materialised sub-matrix of A over global ids (Table 4) behind
    the gs_matrix_* C ABI; every operator runs in ops.cu."""

    def __init__(self, handle, keep=None):
        self._h = handle
        self._keep = keep

    @staticmethod
    def slice_columns(g: "Graph", cols: torch.Tensor, stream=None) -> "Matrix":
        """A[:, cols]."""
        L = load_library()
        _drain()
        cols = cols.to(torch.int32).contiguous()
        h = ctypes.c_void_p()
        _check(L.gs_matrix_slice_columns(g.handle, _ptr(cols), cols.numel(), _stream_ptr(stream),
                                         ctypes.byref(h)), "gs_matrix_slice_columns")
        return Matrix(h, g)

    def slice_rows(self, rows: torch.Tensor, stream=None) -> "Matrix":
        """A[rows, :]."""
        rows = rows.to(torch.int32).contiguous()
        h = ctypes.c_void_p()
        _check(_lib.gs_matrix_slice_rows(self._h, _ptr(rows), rows.numel(), _stream_ptr(stream),
                                         ctypes.byref(h)), "gs_matrix_slice_rows")
        return Matrix(h, self._keep)

    def view(self) -> dict:
        v = _MatrixView()
        _check(_lib.gs_matrix_get_view(self._h, ctypes.byref(v)), "gs_matrix_get_view")
        return {"num_nodes": v.num_nodes,
                "cols": _dev_tensor(v.cols, v.n_cols, torch.int32, self),
                "indptr": _dev_tensor(v.indptr, v.n_cols + 1, torch.int64, self),
                "row": _dev_tensor(v.row, v.nnz, torch.int32, self),
                "eid": _dev_tensor(v.eid, v.nnz, torch.int64, self),
                "val": _dev_tensor(v.val, v.nnz, torch.float32, self)}

    def sum(self, axis: int, stream=None) -> torch.Tensor:
        """A.sum(axis): axis 0 per column, axis 1 dense per global row id."""
        v = self.view()
        n = v["cols"].numel() if axis == 0 else v["num_nodes"]
        out = torch.empty(n, dtype=torch.float32, device="cuda")
        _check(_lib.gs_matrix_sum(self._h, int(axis), _ptr(out), _stream_ptr(stream)), "gs_matrix_sum")
        return out

    def broadcast_(self, op: int, V: torch.Tensor, axis: int, stream=None) -> "Matrix":
        """A.<op>(V, axis), in place."""
        V = V.to(torch.float32).contiguous()
        _check(_lib.gs_matrix_broadcast(self._h, int(op), _ptr(V), int(axis), _stream_ptr(stream)),
               "gs_matrix_broadcast")
        self._V = V
        return self

    def elementwise_(self, op: int, x: float, stream=None) -> "Matrix":
        """A <op> x, in place."""
        _check(_lib.gs_matrix_elementwise(self._h, int(op), float(x), _stream_ptr(stream)),
               "gs_matrix_elementwise")
        return self

    def individual_sample(self, K: int, use_values=False, replace=False, rng_key=0, layer=0, batch_index=0,
                          stream=None) -> "Matrix":
        """A.individual_sample(K, probs) (probs = the values when use_values)."""
        h = ctypes.c_void_p()
        _check(_lib.gs_matrix_individual_sample(self._h, int(K), int(bool(use_values)), int(bool(replace)),
                                                ctypes.c_uint64(rng_key), int(layer), int(batch_index),
                                                _stream_ptr(stream), ctypes.byref(h)),
               "gs_matrix_individual_sample")
        return Matrix(h, self._keep)

    def collective_sample(self, K: int, node_probs: torch.Tensor = None, rng_key=0, layer=0, batch_index=0,
                          stream=None) -> "Matrix":
        """A.collective_sample(K, node_probs) (node_probs: dense float per global id, or None)."""
        h = ctypes.c_void_p()
        p = None if node_probs is None else node_probs.to(torch.float32).contiguous()
        _check(_lib.gs_matrix_collective_sample(self._h, int(K), None if p is None else _ptr(p),
                                                ctypes.c_uint64(rng_key), int(layer), int(batch_index),
                                                _stream_ptr(stream), ctypes.byref(h)),
               "gs_matrix_collective_sample")
        return Matrix(h, self._keep)

    def map_reduce(self, ops, scalars, axis=None, stream=None):
        """Fused element-wise chain; axis None: in place (returns self), 0/1: the sums."""
        o = (ctypes.c_int * len(ops))(*[int(x) for x in ops])
        sc = (ctypes.c_float * len(scalars))(*[float(x) for x in scalars])
        if axis is None:
            _check(_lib.gs_matrix_map_reduce(self._h, o, sc, len(ops), -1, None, _stream_ptr(stream)),
                   "gs_matrix_map_reduce")
            return self
        v = self.view()
        n = v["cols"].numel() if axis == 0 else v["num_nodes"]
        out = torch.empty(n, dtype=torch.float32, device="cuda")
        _check(_lib.gs_matrix_map_reduce(self._h, o, sc, len(ops), int(axis), _ptr(out), _stream_ptr(stream)),
               "gs_matrix_map_reduce")
        return out

    def asgcn_bias(self, X: torch.Tensor, wg: torch.Tensor, stream=None) -> torch.Tensor:
        """AS-GCN-style node bias (R30): dense float[num_nodes]."""
        X = X.to(torch.bfloat16).contiguous()
        wg = wg.to(torch.float32).contiguous()
        out = torch.empty(self.view()["num_nodes"], dtype=torch.float32, device="cuda")
        _check(_lib.gs_matrix_asgcn_bias(self._h, _ptr(X), X.shape[1], _ptr(wg), _ptr(out), _stream_ptr(stream)),
               "gs_matrix_asgcn_bias")
        return out

    def row_ids(self, stream=None) -> torch.Tensor:
        """A.row(): distinct row ids ascending."""
        v = self.view()
        out = torch.empty(max(1, min(v["row"].numel(), v["num_nodes"])), dtype=torch.int32, device="cuda")
        n = ctypes.c_int64()
        _check(_lib.gs_matrix_row_ids(self._h, _ptr(out), ctypes.byref(n), _stream_ptr(stream)),
               "gs_matrix_row_ids")
        return out[:n.value]

    def __del__(self):
        try:
            if getattr(self, "_h", None) and self._h.value and _alive():
                _pending.append(("m", self._h))
                self._h = None
        except TypeError:  # interpreter shutdown: module globals already cleared
            pass


def sample_pinsage(g: Graph, seeds: torch.Tensor, topk, num_walks: int, walk_length: int,
                   restart_prob: float, batch_size=None, batch_index_base=0, rng_key=0,
                   stream=None, out: Blocks = None):
    """PinSAGE-style sampling (Table 2; DESIGN R27) through gs_sample_pinsage."""
    L = load_library()
    _drain()
    seeds = seeds.to(torch.int32).contiguous()
    bs = int(batch_size or max(1, seeds.numel()))
    out = out or Blocks()
    _check(L.gs_sample_pinsage(g.handle, _ptr(seeds), seeds.numel(), bs, int(batch_index_base),
                               _host_i32(topk), len(topk), int(num_walks), int(walk_length),
                               float(restart_prob), ctypes.c_uint64(rng_key), _stream_ptr(stream),
                               ctypes.byref(out._h)), "gs_sample_pinsage")
    out.synced = False
    out._seeds = seeds
    return out


def sample_saint_rw(g: Graph, roots: torch.Tensor, walk_length: int, batch_size=None,
                    batch_index_base=0, rng_key=0, stream=None, out: Blocks = None, retry=True):
    """GraphSAINT-RW (Table 2; DESIGN R26) through gs_sample_saint_rw:
    one induced block per batch of roots."""
    L = load_library()
    _drain()
    roots = roots.to(torch.int32).contiguous()
    bs = int(batch_size or max(1, roots.numel()))
    out = out or Blocks()
    for attempt in range(3):
        _check(L.gs_sample_saint_rw(g.handle, _ptr(roots), roots.numel(), bs, int(batch_index_base),
                                    int(walk_length), ctypes.c_uint64(rng_key), _stream_ptr(stream),
                                    ctypes.byref(out._h)), "gs_sample_saint_rw")
        out.synced = False
        if not retry:
            break
        try:
            out.sync()
            break
        except GSError as e:
            if e.status != 7 or attempt == 2:
                raise
    out._seeds = roots
    return out


def sample_layerwise(g: Graph, seeds: torch.Tensor, n_per_layer, batch_size=None,
                     batch_index_base=0, prob_mode=LADIES, rng_key=0, stream=None,
                     out: Blocks = None, retry=True):
    L = load_library()
    _drain()
    seeds = seeds.to(torch.int32).contiguous()
    bs = int(batch_size or max(1, seeds.numel()))
    out = out or Blocks()
    f = _host_i32(n_per_layer)
    for attempt in range(3):
        _check(L.gs_sample_layerwise(g.handle, _ptr(seeds), seeds.numel(), bs,
                                     int(batch_index_base), f, len(n_per_layer), int(prob_mode),
                                     ctypes.c_uint64(rng_key), _stream_ptr(stream),
                                     ctypes.byref(out._h)), "gs_sample_layerwise")
        out.synced = False
        if not retry:
            break
        try:
            out.sync()
            break
        except GSError as e:
            if e.status != 7 or attempt == 2:
                raise
    out._seeds = seeds
    return out


def random_walk(g: Graph, starts: torch.Tensor, length: int, p=1.0, q=1.0, walker_index_base=0,
                rng_key=0, force_node2vec=False, stream=None, out: torch.Tensor = None):
    """DeepWalk / Node2Vec; returns int32 traces [num_walkers, length + 1] on the device."""
    L = load_library()
    _drain()
    starts = starts.to(torch.int32).contiguous()
    if out is None:
        out = torch.empty((starts.numel(), length + 1), dtype=torch.int32, device=starts.device)
    _check(L.gs_random_walk(g.handle, _ptr(starts), starts.numel(), int(walker_index_base),
                            int(length), float(p), float(q), ctypes.c_uint64(rng_key),
                            WALK_FORCE_NODE2VEC if force_node2vec else 0, _stream_ptr(stream),
                            _ptr(out)), "gs_random_walk")
    return out


def walk_check(g: Graph, stream=None):
    _check(load_library().gs_walk_check(g.handle, _stream_ptr(stream)), "gs_walk_check")


def kernel_launches() -> int:
    """Cumulative number of kernels the library enqueued from this thread
    (gs_kernel_launches); the difference around a call = its launches."""
    return int(load_library().gs_kernel_launches())


def set_profiling(on: bool) -> None:
    """gs_set_profiling: per-kernel event timing of the node-wise sampler."""
    _check(load_library().gs_set_profiling(int(bool(on))), "gs_set_profiling")


def blocks_profile(b: "Blocks") -> list:
    """[(kernel, ms)] of the call that produced b (profiling on), gs_blocks_profile."""
    L = load_library()
    res, i = [], 0
    name, ms = ctypes.c_char_p(), ctypes.c_double()
    while b._h and L.gs_blocks_profile(b._h, i, ctypes.byref(name), ctypes.byref(ms)) == 0:
        res.append((name.value.decode(), ms.value))
        i += 1
    return res


class HeteroSample:
    """Result of sample_neighbors_hetero: blocks[l][r] (Matrix views, None when
    skipped) and frontiers[l][t] (device int32), l = 0 .. num_layers."""

    def __init__(self, h, L, R, T, keep):
        self._h = h
        self._keep = keep
        self.blocks, self.frontiers = [], []
        for l in range(L):
            row = []
            for r in range(R):
                m = ctypes.c_void_p()
                _check(_lib.gs_hetero_block(h, l, r, ctypes.byref(m)), "gs_hetero_block")
                row.append(self._view(m) if m.value else None)
            self.blocks.append(row)
        for l in range(L + 1):
            fl = []
            for t in range(T):
                p, n = ctypes.c_void_p(), ctypes.c_int64()
                _check(_lib.gs_hetero_frontier(h, l, t, ctypes.byref(p), ctypes.byref(n)), "gs_hetero_frontier")
                fl.append(_dev_tensor(p.value, n.value, torch.int32, self))
            self.frontiers.append(fl)

    def _view(self, m):  # a borrowed gs_matrix (owned by the gs_hetero)
        v = _MatrixView()
        _check(_lib.gs_matrix_get_view(m, ctypes.byref(v)), "gs_matrix_get_view")
        return {"num_nodes": v.num_nodes,
                "cols": _dev_tensor(v.cols, v.n_cols, torch.int32, self),
                "indptr": _dev_tensor(v.indptr, v.n_cols + 1, torch.int64, self),
                "row": _dev_tensor(v.row, v.nnz, torch.int32, self),
                "eid": _dev_tensor(v.eid, v.nnz, torch.int64, self)}

    def __del__(self):
        try:
            if getattr(self, "_h", None) and _alive():
                _lib.gs_hetero_destroy(self._h)
                self._h = None
        except TypeError:
            pass


def sample_neighbors_hetero(relations, num_nodes, seeds, fanouts, rng_key=0, stream=None) -> HeteroSample:
    """Heterogeneous node-wise sampling (gs_sample_neighbors_hetero).
    relations: list of (src_type, dst_type, Graph); num_nodes[t]; seeds[t]
    (device int32, possibly empty); fanouts[l][r]."""
    L = load_library()
    _drain()
    R, T, NL = len(relations), len(num_nodes), len(fanouts)
    garr = (ctypes.c_void_p * R)(*[g.handle.value for _, _, g in relations])
    st = torch.tensor([s for s, _, _ in relations], dtype=torch.int32)
    dt = torch.tensor([d for _, d, _ in relations], dtype=torch.int32)
    nn = torch.tensor(list(num_nodes), dtype=torch.int64)
    sd = [s.to(torch.int32).contiguous() for s in seeds]
    sarr = (ctypes.c_void_p * T)(*[(s.data_ptr() if s.numel() else None) for s in sd])
    ns = torch.tensor([s.numel() for s in sd], dtype=torch.int64)
    fo = torch.tensor([int(k) for fl in fanouts for k in fl], dtype=torch.int32)
    h = ctypes.c_void_p()
    _check(L.gs_sample_neighbors_hetero(garr, _ptr(st), _ptr(dt), R, T, _ptr(nn), sarr, _ptr(ns), _ptr(fo), NL,
                                        ctypes.c_uint64(rng_key), _stream_ptr(stream), ctypes.byref(h)),
           "gs_sample_neighbors_hetero")
    return HeteroSample(h, NL, R, T, (relations, sd))
