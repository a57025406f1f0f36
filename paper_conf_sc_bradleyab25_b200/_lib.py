"""ctypes binding of ``libfsgc.so`` (include/fsgc.h).  Argument marshalling
only: every step of the counting path runs in the library's CUDA kernels.

The library is loaded eagerly and the import FAILS LOUDLY if it is missing:
there is no CPU fallback.
"""
import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libfsgc.so")

FSGC_OK = 0
FSGC_ERR_INVALID = 1
FSGC_ERR_CUDA = 2
FSGC_ERR_OOM = 3
FSGC_ERR_PATTERN = 4
FSGC_ERR_INTERNAL = 5
FSGC_MAX_PATTERN_VERTICES = 64
FSGC_MAX_CORE = 8
FSGC_MAX_VENN_BITS = 6
FSGC_MAX_BATCH = 16
FSGC_FLAG_NO_DEGREE_FILTER = 1
FSGC_FLAG_SHARD_SUPPORT = 2
FSGC_STAGE_SUPPORT = 1
FSGC_STAGE_COUNT = 2
FSGC_STAGE_ALL = 3

EXPORTS = [
    "fsgc_load_graph", "fsgc_graph_get_info", "fsgc_graph_download", "fsgc_free_graph",
    "fsgc_compile_pattern", "fsgc_pattern_get_info", "fsgc_free_pattern",
    "fsgc_count", "fsgc_num_roots", "fsgc_finalize", "fsgc_last_error", "fsgc_version",
    "fsgc_plan_create", "fsgc_plan_workspace_bytes", "fsgc_plan_enqueue", "fsgc_plan_decode",
    "fsgc_plan_free", "fsgc_plan_enqueue_stage", "fsgc_plan_support_region",
]


class FsgcError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"fsgc error {code}: {msg}")
        self.code = code


class u128(C.Structure):
    _fields_ = [("lo", C.c_uint64), ("hi", C.c_uint64)]

    @property
    def value(self):
        return (self.hi << 64) | self.lo

    @staticmethod
    def of(v):
        return u128(v & ((1 << 64) - 1), v >> 64)


class GraphInfo(C.Structure):
    _fields_ = [
        ("num_vertices", C.c_int64), ("num_edges", C.c_int64), ("max_degree", C.c_int64),
        ("offsets", C.c_void_p), ("adj", C.c_void_p), ("row", C.c_void_p),
        ("osrc", C.c_void_p), ("odst", C.c_void_p), ("order", C.c_void_p),
    ]


class PatternInfo(C.Structure):
    _fields_ = [
        ("num_vertices", C.c_int), ("num_edges", C.c_int), ("core_size", C.c_int),
        ("core_order", C.c_int32 * FSGC_MAX_CORE), ("num_types", C.c_int),
        ("type_anchor", C.c_uint64 * FSGC_MAX_PATTERN_VERTICES),
        ("type_count", C.c_int32 * FSGC_MAX_PATTERN_VERTICES),
        ("core_mask", C.c_uint64), ("aut", C.c_uint64), ("aut_core", C.c_uint64),
        ("aut_core_labeled", C.c_uint64), ("fringe_factorial", C.c_uint64),
    ]


class Result(C.Structure):
    _fields_ = [
        ("count", u128), ("raw", u128), ("divisor", C.c_uint64), ("core_matches", C.c_uint64),
        ("overflow", C.c_int32), ("root_pattern_vertex", C.c_int32),
        ("kernel_ms", C.c_float), ("aux_ms", C.c_float), ("kernel_launches", C.c_int32),
        ("pass_index", C.c_int32), ("pass_kind", C.c_int32),
    ]


class CountOpts(C.Structure):
    _fields_ = [
        ("root_begin", C.c_int64), ("root_end", C.c_int64), ("shard_index", C.c_int32),
        ("shard_count", C.c_int32), ("no_symmetry_breaking", C.c_int32), ("flags", C.c_int32),
    ]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"{LIB_PATH} is missing: build it with `python paper_conf_sc_bradleyab25_b200/build.py` "
            "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    vp, i64, i32 = C.c_void_p, C.c_int64, C.c_int32
    sig = {
        "fsgc_load_graph": ([vp, i64, C.c_int, i64, C.c_int, vp, C.POINTER(vp)], C.c_int),
        "fsgc_graph_get_info": ([vp, C.POINTER(GraphInfo)], C.c_int),
        "fsgc_graph_download": ([vp, vp, vp, vp], C.c_int),
        "fsgc_free_graph": ([vp], None),
        "fsgc_compile_pattern": ([C.c_int, vp, C.c_int, vp, C.c_int, C.POINTER(vp)], C.c_int),
        "fsgc_pattern_get_info": ([vp, C.POINTER(PatternInfo)], C.c_int),
        "fsgc_free_pattern": ([vp], None),
        "fsgc_count": ([vp, vp, C.c_int, C.POINTER(CountOpts), C.POINTER(Result), vp], C.c_int),
        "fsgc_num_roots": ([vp, vp, C.c_int, C.POINTER(i64)], C.c_int),
        "fsgc_finalize": ([u128, C.c_uint64, i32, C.POINTER(u128), C.POINTER(i32)], C.c_int),
        "fsgc_plan_create": ([vp, vp, C.c_int, C.POINTER(CountOpts), C.POINTER(vp)], C.c_int),
        "fsgc_plan_workspace_bytes": ([vp, C.POINTER(C.c_size_t), C.POINTER(C.c_size_t)], C.c_int),
        "fsgc_plan_enqueue": ([vp, vp, vp, vp], C.c_int),
        "fsgc_plan_enqueue_stage": ([vp, vp, vp, C.c_int, vp], C.c_int),
        "fsgc_plan_support_region": ([vp, C.POINTER(C.c_size_t), C.POINTER(i64)], C.c_int),
        "fsgc_plan_decode": ([vp, vp, C.POINTER(Result)], C.c_int),
        "fsgc_plan_free": ([vp], None),
        "fsgc_last_error": ([], C.c_char_p),
        "fsgc_version": ([], C.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


lib = _load()


def check(rc):
    if rc != FSGC_OK:
        raise FsgcError(rc, lib.fsgc_last_error().decode())
    return rc
