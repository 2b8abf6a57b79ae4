"""ctypes declarations of include/ug.h (argument marshalling only; no computation here).

The product path has NO fallback: if libugraph.so is missing or fails to load, importing
this module raises.  Build it with `make` (or __graft_entry__.build()).
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("UG_LIBRARY") or os.path.join(_HERE, "libugraph.so")   # override: experiments only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libugraph.so not built at {LIB_PATH}: run `make` in the repo root "
                      "(there is no CPU fallback for the graph operator)")
lib = ctypes.CDLL(LIB_PATH)

UG_OK = 0
STATUS = {0: "UG_OK", 1: "UG_ERR_INVALID_ARG", 2: "UG_ERR_UNSUPPORTED_OP", 3: "UG_ERR_SHAPE",
          4: "UG_ERR_INDEX_RANGE", 5: "UG_ERR_ALIGNMENT", 6: "UG_ERR_OOM", 7: "UG_ERR_CUDA",
          8: "UG_ERR_UNSUPPORTED_SCHEDULE"}

EDGE_OPS = {"copy_lhs": 0, "copy_rhs": 1, "add": 2, "sub": 3, "mul": 4, "div": 5, "dot": 6}
GATHER_OPS = {"assign": 0, "copy_rhs": 0, "sum": 1, "max": 2, "min": 3, "mean": 4}
TTYPES = {None: 0, "null": 0, "NULL": 0, "u": 1, "Src_V": 1, "v": 2, "Dst_V": 2, "e": 3, "Edge": 3}
STRATEGIES = {"AUTO": 0, "TV": 1, "TE": 2, "WV": 3, "WE": 4, "BV": 5, "BE": 6, "SV": 7}
UG_GRAPH_HOST_ONLY = 1


class UgTensor(ctypes.Structure):
    _fields_ = [("data", ctypes.c_void_p), ("type", ctypes.c_int32), ("width", ctypes.c_int32),
                ("ld", ctypes.c_int64)]


class UgOpInfo(ctypes.Structure):
    _fields_ = [("edge_op", ctypes.c_int32), ("gather_op", ctypes.c_int32), ("A", UgTensor),
                ("B", UgTensor), ("C", UgTensor), ("feat", ctypes.c_int32), ("heads", ctypes.c_int32)]


class UgSchedule(ctypes.Structure):
    _fields_ = [("strategy", ctypes.c_int32), ("group", ctypes.c_int32), ("tile", ctypes.c_int32),
                ("block_threads", ctypes.c_int32), ("ftile", ctypes.c_int32), ("vec", ctypes.c_int32),
                ("flags", ctypes.c_int32)]


class UgAllocator(ctypes.Structure):
    _fields_ = [("alloc", ctypes.c_void_p), ("free", ctypes.c_void_p), ("ctx", ctypes.c_void_p)]


_p = ctypes.c_void_p
_i64 = ctypes.c_int64
_i32 = ctypes.c_int32
_st = ctypes.c_int
_gpp = ctypes.POINTER(ctypes.c_void_p)

SIGNATURES = {
    "ug_graph_create": ([_i64, _i64, _p, _p, ctypes.c_int, ctypes.c_int, _p, _p, _gpp], _st),
    "ug_graph_create_csr": ([_i64, _i64, _p, _p, _p, ctypes.c_int, ctypes.c_int, _p, _p, _gpp], _st),
    "ug_graph_destroy": ([_p], _st),
    "ug_graph_stats": ([_p, _p, _p, _p, _p, _p], _st),
    "ug_graph_csr": ([_p, _p, _p, _p], _st),
    "ug_graph_partition": ([_p, _i32, _p], _st),
    "ug_graph_view_rows": ([_p, _i64, _i64, _gpp], _st),
    "ug_op_validate": ([_p, ctypes.POINTER(UgOpInfo)], _st),
    "ug_schedule_select": ([_p, ctypes.POINTER(UgOpInfo), ctypes.POINTER(UgSchedule)], _st),
    "ug_selector_load": ([ctypes.c_char_p], _st),
    "ug_selector_load_model": ([ctypes.c_char_p], _st),
    "ug_op_run": ([_p, ctypes.POINTER(UgOpInfo), ctypes.POINTER(UgSchedule), _p], _st),
    "ug_op_run_events": ([_p, ctypes.POINTER(UgOpInfo), ctypes.POINTER(UgSchedule), _p, _p, _p], _st),
    "ug_op_launch_count": ([_p, ctypes.POINTER(UgOpInfo), ctypes.POINTER(UgSchedule),
                            ctypes.POINTER(ctypes.c_int32)], _st),
    "ug_edge_permute": ([_p, _p, _p, _i32, _p], _st),
    "ug_gat_attention": ([_p, _p, _i64, _p, _i64, _p, _i64, _i32, _i32, ctypes.c_float, _p, _i64, _p, _i64, _p],
                         _st),
    "ug_scratch_trim": ([], _st),
    "ug_dot_attention": ([_p, _p, _i64, _p, _i64, _p, _i64, _i32, _i32, _i32, ctypes.c_float, _p, _i64, _p, _i64,
                          _p], _st),
    "ug_op_run_arg": ([_p, ctypes.POINTER(UgOpInfo), _p, _i64, _p], _st),
    "ug_arg_scatter": ([_p, _p, _i64, _i32, _p, _i64, _i32, _p, _i64, _i32, _p], _st),
    "ug_graph_reorder": ([_p, _i32, _p], _st),
    "ug_rows_gather": ([_p, _i64, _p, _i64, _i32, _p, _i64, _p], _st),
    "ug_schedule_parse": ([ctypes.c_char_p, ctypes.POINTER(UgSchedule)], _st),
    "ug_schedule_format": ([ctypes.POINTER(UgSchedule), ctypes.c_char_p, ctypes.c_size_t], _st),
    "ug_status_string": ([_st], ctypes.c_char_p),
    "ug_last_error": ([], ctypes.c_char_p),
    "ug_version": ([], ctypes.c_char_p),
}

for _name, (_args, _res) in SIGNATURES.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = _res


class UgError(RuntimeError):
    def __init__(self, status, where):
        self.status = STATUS.get(status, str(status))
        detail = lib.ug_last_error().decode()
        super().__init__(f"{where}: {self.status}: {detail}")


def check(status, where):
    if status != UG_OK:
        raise UgError(status, where)
