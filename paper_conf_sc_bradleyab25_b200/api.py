"""Python face of the C ABI (include/fsgc.h): same names, argument marshalling
only.  PyTorch is used for streams, device tensors and torch.distributed.

    g = fsgc_load_graph(edges, n)                       # numpy / torch edges
    p = fsgc_compile_pattern(n_p, pattern_edges)        # Sec. 3.4 decomposition
    res = fsgc_count(g, [p])                            # exact counts (ints)
    res = fsgc_count_distributed(g, [p])                # shard roots over ranks,
                                                        # one all-reduce of the
                                                        # 128-bit partial sums
"""
import ctypes as C
from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

from . import _lib
from ._lib import lib, check, CountOpts, GraphInfo, PatternInfo, Result, u128


def _stream_handle(stream):
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return C.c_void_p(torch.cuda.current_stream().cuda_stream)
        except ImportError:
            pass
        return C.c_void_p(0)
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


class Graph:
    """Device-resident degree-ordered CSR (owns the fsgc_graph handle)."""

    def __init__(self, handle):
        self._h = C.c_void_p(handle)
        info = GraphInfo()
        check(lib.fsgc_graph_get_info(self._h, C.byref(info)))
        self.info = info
        self.n = info.num_vertices
        self.m = info.num_edges
        self.max_degree = info.max_degree
        self._plans = {}          # distributed plans of this graph (freed with it)

    @property
    def handle(self):
        return self._h

    def download(self):
        """(offsets int64[n+1], adj int32[2m], order int32[n]) on the host."""
        offs = np.empty(self.n + 1, dtype=np.int64)
        adj = np.empty(max(2 * self.m, 1), dtype=np.int32)
        order = np.empty(self.n, dtype=np.int32)
        check(lib.fsgc_graph_download(self._h, offs.ctypes.data, adj.ctypes.data, order.ctypes.data))
        return offs, adj[:2 * self.m], order

    def free(self):
        for plan in getattr(self, "_plans", {}).values():
            plan.free()
        self._plans = {}
        if self._h:
            lib.fsgc_free_graph(self._h)
            self._h = C.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Pattern:
    """Compiled pattern (owns the fsgc_pattern handle)."""

    def __init__(self, handle, name=""):
        self._h = C.c_void_p(handle)
        self.name = name
        info = PatternInfo()
        check(lib.fsgc_pattern_get_info(self._h, C.byref(info)))
        self.info = info
        self.core_order = [info.core_order[i] for i in range(info.core_size)]
        self.core = sorted(self.core_order)
        self.types = [(frozenset(v for v in range(64) if info.type_anchor[t] >> v & 1), info.type_count[t])
                      for t in range(info.num_types)]
        self.aut = info.aut
        self.aut_core = info.aut_core
        self.aut_core_labeled = info.aut_core_labeled
        self.fringe_factorial = info.fringe_factorial

    @property
    def handle(self):
        return self._h

    def free(self):
        if self._h:
            lib.fsgc_free_pattern(self._h)
            self._h = C.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


@dataclass
class CountResult:
    count: Optional[int]      # None if overflow or partial
    raw: int
    divisor: int
    core_matches: int
    overflow: bool
    root_pattern_vertex: int
    kernel_ms: float = 0.0
    aux_ms: float = 0.0
    kernel_launches: int = 0
    pass_index: int = 0
    pass_kind: int = 0


def fsgc_load_graph(edges, num_vertices, stream=None) -> Graph:
    """edges: numpy [E,2] int32/int64 (host, pinned or pageable) or a torch
    tensor [E,2] int32/int64 on the host or on the current CUDA device."""
    try:
        import torch
    except ImportError:  # pragma: no cover
        torch = None
    on_device = 0
    if torch is not None and isinstance(edges, torch.Tensor):
        if edges.dtype not in (torch.int32, torch.int64):
            raise TypeError("edges must be int32 or int64")
        edges = edges.contiguous()
        ptr, E, ib = edges.data_ptr(), edges.shape[0], edges.element_size()
        on_device = 1 if edges.is_cuda else 0
        keep = edges
    else:
        arr = np.ascontiguousarray(edges)
        if arr.dtype not in (np.int32, np.int64):
            arr = arr.astype(np.int64)
        arr = arr.reshape(-1, 2)
        ptr, E, ib = arr.ctypes.data, arr.shape[0], arr.itemsize
        keep = arr
    h = C.c_void_p()
    check(lib.fsgc_load_graph(C.c_void_p(ptr), int(E), int(ib), int(num_vertices), on_device,
                              _stream_handle(stream), C.byref(h)))
    del keep
    return Graph(h.value)


def fsgc_compile_pattern(num_vertices, edges, core=None, name="") -> Pattern:
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.int32).reshape(-1, 2))
    c = None if core is None else np.ascontiguousarray(np.asarray(core, dtype=np.int32))
    h = C.c_void_p()
    check(lib.fsgc_compile_pattern(int(num_vertices), e.ctypes.data if e.size else None, e.shape[0],
                                   c.ctypes.data if c is not None else None,
                                   0 if c is None else c.size, C.byref(h)))
    return Pattern(h.value, name)


def compile_named(p) -> Pattern:
    """compile an ``inputs.patterns.Pattern``"""
    return fsgc_compile_pattern(p.n, list(p.edges), p.core, p.name)


def _opts(root_begin=0, root_end=-1, shard_index=0, shard_count=1, no_symmetry_breaking=False,
          no_degree_filter=False, shard_support=False):
    o = CountOpts()
    o.root_begin = root_begin
    o.root_end = root_end
    o.shard_index = shard_index
    o.shard_count = shard_count
    o.no_symmetry_breaking = 1 if no_symmetry_breaking else 0
    o.flags = ((_lib.FSGC_FLAG_NO_DEGREE_FILTER if no_degree_filter else 0) |
               (_lib.FSGC_FLAG_SHARD_SUPPORT if shard_support else 0))
    return o


def fsgc_count(graph: Graph, patterns: Sequence[Pattern], stream=None, **kw) -> List[CountResult]:
    """Count every pattern (exact ints).  kw: root_begin, root_end,
    shard_index, shard_count, no_symmetry_breaking, no_degree_filter."""
    pats = list(patterns)
    arr = (C.c_void_p * len(pats))(*[p.handle.value for p in pats])
    res = (Result * len(pats))()
    o = _opts(**kw)
    check(lib.fsgc_count(graph.handle, arr, len(pats), C.byref(o), res, _stream_handle(stream)))
    return _results(res, o.shard_count == 1 and o.root_begin <= 0 and o.root_end < 0)


def _results(res, whole):
    out = []
    for r in res:
        out.append(CountResult(
            count=(r.count.value if (whole and not r.overflow) else None), raw=r.raw.value,
            divisor=r.divisor, core_matches=r.core_matches, overflow=bool(r.overflow),
            root_pattern_vertex=r.root_pattern_vertex, kernel_ms=r.kernel_ms, aux_ms=r.aux_ms,
            kernel_launches=r.kernel_launches, pass_index=r.pass_index, pass_kind=r.pass_kind))
    return out


class Plan:
    """fsgc_plan: a reusable, CUDA-graph-capturable count.

        plan = fsgc_plan_create(g, pats)
        plan.enqueue(stream)          # async; capturable
        torch.cuda.synchronize()
        results = plan.decode()
    The plan owns its device workspace and a pinned host result block."""

    def __init__(self, graph, patterns, **kw):
        import torch
        self.graph = graph
        self.patterns = list(patterns)
        arr = (C.c_void_p * len(self.patterns))(*[p.handle.value for p in self.patterns])
        self._opts = _opts(**kw)
        self.whole = self._opts.shard_count == 1 and self._opts.root_begin <= 0 and self._opts.root_end < 0
        h = C.c_void_p()
        check(lib.fsgc_plan_create(graph.handle, arr, len(self.patterns), C.byref(self._opts), C.byref(h)))
        self._h = h
        ws, raw = C.c_size_t(), C.c_size_t()
        check(lib.fsgc_plan_workspace_bytes(self._h, C.byref(ws), C.byref(raw)))
        self.workspace = torch.empty(max(ws.value, 1), dtype=torch.uint8, device="cuda")
        self.raw = torch.empty(max(raw.value, 1), dtype=torch.uint8).pin_memory()
        self.workspace_bytes, self.raw_bytes = ws.value, raw.value

    def enqueue(self, stream=None):
        check(lib.fsgc_plan_enqueue(self._h, C.c_void_p(self.workspace.data_ptr()),
                                    C.c_void_p(self.raw.data_ptr()), _stream_handle(stream)))

    def enqueue_stage(self, stages, stream=None):
        """stages: FSGC_STAGE_SUPPORT | FSGC_STAGE_COUNT bit mask"""
        check(lib.fsgc_plan_enqueue_stage(self._h, C.c_void_p(self.workspace.data_ptr()),
                                          C.c_void_p(self.raw.data_ptr()), int(stages),
                                          _stream_handle(stream)))

    def support(self):
        """the plan's per-edge support array as an int32 view of the
        workspace (None when no pass reads it)"""
        off, cnt = C.c_size_t(), C.c_int64()
        check(lib.fsgc_plan_support_region(self._h, C.byref(off), C.byref(cnt)))
        if cnt.value == 0:
            return None
        return self.workspace[off.value:off.value + 4 * cnt.value].view(dtype=__import__("torch").int32)

    def decode(self) -> List[CountResult]:
        res = (Result * len(self.patterns))()
        check(lib.fsgc_plan_decode(self._h, C.c_void_p(self.raw.data_ptr()), res))
        return _results(res, self.whole)

    def free(self):
        if getattr(self, "_h", None):
            lib.fsgc_plan_free(self._h)
            self._h = C.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def fsgc_plan_create(graph: Graph, patterns: Sequence[Pattern], **kw) -> Plan:
    return Plan(graph, patterns, **kw)


def fsgc_num_roots(graph: Graph, pattern: Pattern, no_symmetry_breaking=False) -> int:
    v = C.c_int64()
    check(lib.fsgc_num_roots(graph.handle, pattern.handle, 1 if no_symmetry_breaking else 0, C.byref(v)))
    return v.value


def fsgc_finalize(raw: int, divisor: int, overflow: bool = False):
    c = u128()
    o = C.c_int32()
    check(lib.fsgc_finalize(u128.of(raw), divisor, 1 if overflow else 0, C.byref(c), C.byref(o)))
    return None if o.value else c.value


def _limbs(values, flags):
    """128-bit values -> int64 tensor of four 32-bit limbs + overflow flag
    each (sums of up to 2^31 ranks cannot overflow an int64 limb)."""
    out = []
    for v, f in zip(values, flags):
        out += [(v >> (32 * i)) & 0xFFFFFFFF for i in range(4)] + [1 if f else 0]
    return out


def _unlimbs(limbs, npats):
    vals, flags = [], []
    for k in range(npats):
        l = limbs[5 * k:5 * k + 5]
        v = sum(int(l[i]) << (32 * i) for i in range(4))
        flags.append(bool(l[4]) or v >> 128 != 0)
        vals.append(v & ((1 << 128) - 1))
    return vals, flags


def combine_partials(part: Sequence[CountResult], group=None, device=None) -> List[CountResult]:
    """All-reduce per-rank partial results (raw 128-bit sums as 32-bit limbs
    in int64, overflow flags, core-match counts) in ONE collective and
    finalise the counts.  ``device``: where the reduction tensor lives
    (a CUDA device for NCCL, CPU for gloo)."""
    import torch
    import torch.distributed as dist
    if device is None:
        device = (torch.device("cuda", torch.cuda.current_device())
                  if dist.get_backend(group) == "nccl" else torch.device("cpu"))
    t = torch.tensor(_limbs([r.raw for r in part], [r.overflow for r in part]) +
                     [r.core_matches for r in part], dtype=torch.int64, device=device)
    dist.all_reduce(t, group=group)
    h = t.cpu().tolist()
    raws, flags = _unlimbs(h, len(part))
    out = []
    for k, r in enumerate(part):
        cnt = None if flags[k] else fsgc_finalize(raws[k], r.divisor, False)
        out.append(CountResult(count=cnt, raw=raws[k], divisor=r.divisor,
                               core_matches=h[5 * len(part) + k], overflow=flags[k],
                               root_pattern_vertex=r.root_pattern_vertex, kernel_ms=r.kernel_ms,
                               aux_ms=r.aux_ms, kernel_launches=r.kernel_launches,
                               pass_index=r.pass_index, pass_kind=r.pass_kind))
    return out


def distributed_plan(graph: Graph, patterns: Sequence[Pattern], rank: int, world: int, **kw) -> Plan:
    """cached plan of this rank's shard: root chunks AND the support pass's
    chunks dealt round-robin (FSGC_FLAG_SHARD_SUPPORT).  The cache lives on
    the graph object and is released by ``Graph.free()``."""
    key = (tuple(p.handle.value for p in patterns), rank, world, tuple(sorted(kw.items())))
    plan = graph._plans.get(key)
    if plan is None:
        if len(graph._plans) >= 16:
            for old in graph._plans.values():
                old.free()
            graph._plans.clear()
        plan = Plan(graph, patterns, shard_index=rank, shard_count=world, shard_support=world > 1, **kw)
        graph._plans[key] = plan
    return plan


def fsgc_count_distributed(graph: Graph, patterns: Sequence[Pattern], group=None, stream=None,
                           **kw) -> List[CountResult]:
    """Strong-scaling count over the ranks of ``group``: the graph is
    replicated in every rank's HBM; the support pass's chunks and the root
    chunks are dealt round-robin (shard = rank).  Two exchanges:
      1. the per-edge support array (int32[m], partial triangle counts of
         each shard) is summed by an all-reduce between the two stages;
      2. the per-rank 128-bit partial sums are combined by ONE all-reduce.
    NCCL over NVLink for CUDA tensors; gloo works too (CUDA tensors are
    staged through the host)."""
    import torch
    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    if world == 1:
        return fsgc_count(graph, patterns, stream=stream, **kw)
    pats = list(patterns)
    plan = distributed_plan(graph, pats, rank, world, **kw)
    st = stream if stream is not None else torch.cuda.current_stream()
    with torch.cuda.stream(st):
        plan.enqueue_stage(_lib.FSGC_STAGE_SUPPORT, st)
        sup = plan.support()
        if sup is not None:
            dist.all_reduce(sup, group=group)
        plan.enqueue_stage(_lib.FSGC_STAGE_COUNT, st)
    st.synchronize()
    return combine_partials(plan.decode(), group)
