"""Thin ctypes binding of libvf.so (include/vf.h) — argument marshalling only.

Every step of the path runs in libvf's CUDA kernels; torch supplies device
memory (tensors' data_ptr()) and streams. There is no CPU fallback: if
libvf.so is missing or no CUDA device is present, constructing a Ctx raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(PKG, "libvf.so")

# enums mirrored from include/vf.h
VF_OK = 0
CUDA, SHAREDOA, COAL, TYPEPTR, CONCORD = 0, 1, 2, 3, 4
VARIANTS = {"cuda": CUDA, "sharedoa": SHAREDOA, "coal": COAL, "typeptr": TYPEPTR, "concord": CONCORD,
            "cuda_packed": CUDA}  # cuda_packed: CUDA dispatch over an index-ordered slab (vf_alloc_packed)
ORDERS = {"random": 0, "sorted": 1, "kperwarp": 2}
APP_MICRO, APP_GOL, APP_GEN, APP_GRAPH = 0, 1, 2, 3
MICRO_APPLY, MICRO_GET = 0, 1
GOL_NEXT, GOL_GET = 0, 1
GEN_NEXT, GEN_GET = 0, 1
GRAPH_BFS_EXPAND, GRAPH_BFS_PROBE, GRAPH_CC_UPDATE, GRAPH_PR_CONTRIB, GRAPH_PR_UPDATE = 0, 1, 2, 3, 4
GRAPH_BFS_PROBE_BITS = 5
NOT_FOUND = 0xFFFFFFFF
VA_BITS = 57
MAX_RANGES = 4096

STATUS = {0: "VF_OK", 1: "VF_ERR_INVALID", 2: "VF_ERR_OOM", 3: "VF_ERR_CUDA", 4: "VF_ERR_TAG_BITS",
          5: "VF_ERR_TOO_MANY_TYPES", 6: "VF_ERR_TABLE_FULL", 7: "VF_ERR_UNSUPPORTED"}

# exported symbols (checked by tests/test_abi.py against include/vf.h)
SYMBOLS = [
    "vf_config_default", "vf_create", "vf_destroy", "vf_status_str", "vf_last_error", "vf_app_info",
    "vf_alloc_typed", "vf_alloc_typed_batch", "vf_alloc_cuda", "vf_alloc_packed", "vf_reset", "vf_range_table",
    "vf_regions", "vf_type_vptrs", "vf_resolve", "vf_verify_types", "vf_dispatch_cuda",
    "vf_dispatch_sharedoa", "vf_dispatch_coal", "vf_dispatch_typeptr", "vf_dispatch",
    "vf_gol_neighbors", "vf_gol_swap", "vf_gen_swap", "vf_checksum_i32", "vf_launch_count", "vf_set_tuning",
    "vf_graph_bfs_init", "vf_iota_u32", "vf_fill_f32", "vf_ray_render", "vf_gol_step", "vf_gen_step", "vf_gen_step_rows", "vf_gol_run", "vf_dispatch_host",
    "vf_dispatch_concord", "vf_micro_branch", "vf_collide_tmp_words", "vf_collide_grid",
    "vf_collide_pack_near", "vf_collide_unpack_near",
]
APP_RAY = 4
APP_TRAF = 5
TRAF_CELL_UPDATE, TRAF_VEH_STEP, TRAF_GET, TRAF_PLACE = 0, 1, 2, 3


APP_NBODY = 6
NBODY_UPDATE, NBODY_GET = 0, 1


class nbody_update_args(ctypes.Structure):
    _fields_ = [("pin_dev", ctypes.c_void_p), ("pout_dev", ctypes.c_void_p), ("N", ctypes.c_uint32),
                ("dt", ctypes.c_float), ("eps2", ctypes.c_float * 3), ("damp", ctypes.c_float)]


class nbody_get_args(ctypes.Structure):
    _fields_ = [("vel_out_dev", ctypes.c_void_p), ("idx_base", ctypes.c_uint32)]


APP_STUT = 7
STUT_FORCE, STUT_MOVE, STUT_GET = 0, 1, 2


class stut_force_args(ctypes.Structure):
    _fields_ = [("pos_dev", ctypes.c_void_p), ("F_dev", ctypes.c_void_p), ("break_ratio", ctypes.c_float)]


class stut_move_args(ctypes.Structure):
    _fields_ = [("pos_dev", ctypes.c_void_p), ("F_dev", ctypes.c_void_p), ("inc_offs_dev", ctypes.c_void_p),
                ("inc_dev", ctypes.c_void_p), ("dt", ctypes.c_float), ("c", ctypes.c_float),
                ("v_pull", ctypes.c_float)]


class stut_get_args(ctypes.Structure):
    _fields_ = [("vel_out_dev", ctypes.c_void_p), ("broken_out_dev", ctypes.c_void_p), ("id_base", ctypes.c_uint32),
                ("spring_base", ctypes.c_uint32)]


APP_COLLIDE = 8
COLLIDE_UPDATE, COLLIDE_MERGE, COLLIDE_GET = 0, 1, 2


class collide_update_args(ctypes.Structure):
    _fields_ = [("P_dev", ctypes.c_void_p), ("Ps_dev", ctypes.c_void_p), ("list_dev", ctypes.c_void_p),
                ("cell_start_dev", ctypes.c_void_p), ("slot_dev", ctypes.c_void_p), ("Pm_dev", ctypes.c_void_p),
                ("Vm_dev", ctypes.c_void_p),
                ("near_dev", ctypes.c_void_p), ("G", ctypes.c_uint32), ("rc", ctypes.c_float),
                ("rc2", ctypes.c_float), ("rm2", ctypes.c_float), ("dt", ctypes.c_float),
                ("eps2", ctypes.c_float * 3), ("damp", ctypes.c_float)]


class collide_merge_args(ctypes.Structure):
    _fields_ = [("Pm_dev", ctypes.c_void_p), ("Vm_dev", ctypes.c_void_p), ("near_dev", ctypes.c_void_p),
                ("P_dev", ctypes.c_void_p)]


class collide_get_args(ctypes.Structure):
    _fields_ = [("vel_out_dev", ctypes.c_void_p), ("idx_base", ctypes.c_uint32)]


class collide_grid_args(ctypes.Structure):
    _fields_ = [("N", ctypes.c_uint32), ("G", ctypes.c_uint32), ("rc", ctypes.c_float),
                ("P_dev", ctypes.c_void_p), ("cell_of_dev", ctypes.c_void_p), ("cell_count_dev", ctypes.c_void_p),
                ("cell_start_dev", ctypes.c_void_p), ("list_dev", ctypes.c_void_p), ("Ps_dev", ctypes.c_void_p),
                ("slot_dev", ctypes.c_void_p), ("tmp_dev", ctypes.c_void_p), ("objs_dev", ctypes.c_void_p), ("id_lo", ctypes.c_uint32),
                ("id_hi", ctypes.c_uint32), ("order_dev", ctypes.c_void_p), ("active_dev", ctypes.c_void_p)]


class collide_near_entry(ctypes.Structure):
    _fields_ = [("id", ctypes.c_uint32), ("near", ctypes.c_int32), ("pad", ctypes.c_uint32 * 2),
                ("Pm", ctypes.c_float * 4), ("Vm", ctypes.c_float * 4)]


class traf_cell_args(ctypes.Structure):
    _fields_ = [("blocked_dev", ctypes.c_void_p), ("occ_next_dev", ctypes.c_void_p), ("t", ctypes.c_uint32)]


class traf_step_args(ctypes.Structure):
    _fields_ = [("occ_dev", ctypes.c_void_p), ("blocked_dev", ctypes.c_void_p), ("occ_next_dev", ctypes.c_void_p),
                ("L", ctypes.c_uint32), ("t", ctypes.c_uint32), ("seed", ctypes.c_uint64),
                ("vmax", ctypes.c_uint32 * 3), ("slow_thr", ctypes.c_uint32 * 3)]


class traf_get_args(ctypes.Structure):
    _fields_ = [("pos_out_dev", ctypes.c_void_p), ("v_out_dev", ctypes.c_void_p), ("occ_dev", ctypes.c_void_p),
                ("L", ctypes.c_uint32), ("id_base", ctypes.c_uint32)]


class VFError(RuntimeError):
    def __init__(self, status, msg=""):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class vf_config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("init_chunk_objs", ctypes.c_uint64),
                ("reserve_va", ctypes.c_int), ("va_window_bytes", ctypes.c_uint64),
                ("cuda_heap_bytes", ctypes.c_uint64)]


class vf_range(ctypes.Structure):
    _fields_ = [("start", ctypes.c_uint64), ("end", ctypes.c_uint64), ("type_id", ctypes.c_uint32),
                ("app", ctypes.c_uint32), ("vptr", ctypes.c_uint64)]


class vf_region(ctypes.Structure):
    _fields_ = [("start", ctypes.c_uint64), ("cap_objs", ctypes.c_uint64),
                ("used_objs", ctypes.c_uint64), ("obj_bytes", ctypes.c_uint32),
                ("type_id", ctypes.c_uint32), ("app", ctypes.c_uint32), ("pad", ctypes.c_uint32)]


class micro_get_args(ctypes.Structure):
    _fields_ = [("out_dev", ctypes.c_void_p)]


class gol_next_args(ctypes.Structure):
    _fields_ = [("nbr_dev", ctypes.c_void_p), ("state_out_dev", ctypes.c_void_p)]


class gol_get_args(ctypes.Structure):
    _fields_ = [("counter_out_dev", ctypes.c_void_p), ("type_out_dev", ctypes.c_void_p)]


class gen_next_args(ctypes.Structure):
    _fields_ = [("nbr_dev", ctypes.c_void_p), ("state_out_dev", ctypes.c_void_p),
                ("born_mask", ctypes.c_uint32), ("survive_mask", ctypes.c_uint32), ("C", ctypes.c_uint32)]


gen_get_args = gol_get_args


APP_GRAPH_EN, APP_EDGE = 9, 10
GRAPH_EN_BFS_EXPAND, GRAPH_EN_CC_UPDATE, GRAPH_EN_PR_INIT, GRAPH_EN_PR_GATHER = 0, 1, 2, 3
EDGE_PULL_PR, EDGE_PULL_LABEL, EDGE_GET = 0, 1, 2


class edge_resolver(ctypes.Structure):
    _fields_ = [("start_dev", ctypes.c_void_p), ("end_dev", ctypes.c_void_p), ("type_dev", ctypes.c_void_p),
                ("vptr_dev", ctypes.c_void_p), ("K", ctypes.c_uint32), ("P", ctypes.c_uint32),
                ("rule", ctypes.c_uint32)]


class graph_en_bfs_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("out_edges_dev", ctypes.c_void_p), ("depth_dev", ctypes.c_void_p),
                ("vobj_dev", ctypes.c_void_p), ("chunk_dev", ctypes.c_void_p), ("next_queue_dev", ctypes.c_void_p),
                ("next_chunk_dev", ctypes.c_void_p), ("next_count_dev", ctypes.c_void_p), ("level", ctypes.c_int32),
                ("C", ctypes.c_uint32), ("er", edge_resolver)]


class graph_en_cc_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("in_edges_dev", ctypes.c_void_p), ("label_in_dev", ctypes.c_void_p),
                ("label_out_dev", ctypes.c_void_p), ("changed_dev", ctypes.c_void_p), ("chunk_dev", ctypes.c_void_p),
                ("C", ctypes.c_uint32), ("b", ctypes.c_uint32), ("er", edge_resolver)]


class graph_en_pr_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("in_edges_dev", ctypes.c_void_p), ("rank_in_dev", ctypes.c_void_p),
                ("rank_out_dev", ctypes.c_void_p), ("contrib_dev", ctypes.c_void_p),
                ("dangling_in_dev", ctypes.c_void_p), ("dangling_out_dev", ctypes.c_void_p),
                ("base", ctypes.c_double), ("d", ctypes.c_double), ("Vd", ctypes.c_double),
                ("chunk_dev", ctypes.c_void_p), ("partial_dev", ctypes.c_void_p), ("counter_dev", ctypes.c_void_p),
                ("C", ctypes.c_uint32), ("b", ctypes.c_uint32), ("er", edge_resolver)]


class edge_args(ctypes.Structure):
    _fields_ = [("contrib_dev", ctypes.c_void_p), ("label_dev", ctypes.c_void_p), ("out_dev", ctypes.c_void_p),
                ("slot", ctypes.c_uint32)]


class graph_bfs_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("col_dev", ctypes.c_void_p), ("depth_dev", ctypes.c_void_p),
                ("vobj_dev", ctypes.c_void_p), ("chunk_dev", ctypes.c_void_p), ("next_queue_dev", ctypes.c_void_p),
                ("next_chunk_dev", ctypes.c_void_p), ("next_count_dev", ctypes.c_void_p), ("level", ctypes.c_int32),
                ("C", ctypes.c_uint32)]


class graph_bfs_bits_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("col_dev", ctypes.c_void_p), ("depth_dev", ctypes.c_void_p),
                ("frontier_dev", ctypes.c_void_p), ("next_dev", ctypes.c_void_p), ("chunk_dev", ctypes.c_void_p),
                ("next_count_dev", ctypes.c_void_p), ("level", ctypes.c_int32), ("C", ctypes.c_uint32)]


class graph_cc_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("col_dev", ctypes.c_void_p), ("label_in_dev", ctypes.c_void_p),
                ("label_out_dev", ctypes.c_void_p), ("changed_dev", ctypes.c_void_p), ("chunk_dev", ctypes.c_void_p),
                ("C", ctypes.c_uint32)]


class graph_pr_args(ctypes.Structure):
    _fields_ = [("offs_dev", ctypes.c_void_p), ("col_dev", ctypes.c_void_p), ("rank_in_dev", ctypes.c_void_p),
                ("rank_out_dev", ctypes.c_void_p), ("contrib_dev", ctypes.c_void_p),
                ("dangling_dev", ctypes.c_void_p), ("base", ctypes.c_double), ("d", ctypes.c_double),
                ("Vd", ctypes.c_double), ("chunk_dev", ctypes.c_void_p), ("partial_dev", ctypes.c_void_p),
                ("counter_dev", ctypes.c_void_p), ("C", ctypes.c_uint32)]


_lib = None


def lib(required: bool = True):
    """Load libvf.so (fails loudly when it is missing: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO):
        raise FileNotFoundError(f"{SO} not built: run __graft_entry__.build()")
    L = ctypes.CDLL(SO)
    P, U32, U64, I = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    sig = {
        "vf_config_default": (None, [ctypes.POINTER(vf_config)]),
        "vf_create": (I, [ctypes.POINTER(vf_config), ctypes.POINTER(P)]),
        "vf_destroy": (None, [P]),
        "vf_status_str": (ctypes.c_char_p, [I]),
        "vf_last_error": (ctypes.c_char_p, [P]),
        "vf_app_info": (I, [U32, ctypes.POINTER(U32), ctypes.POINTER(U32), ctypes.POINTER(U32)]),
        "vf_alloc_typed": (I, [P, U32, U32, U64, P, U32, P, I, P]),
        "vf_alloc_typed_batch": (I, [P, U32, P, U64, P, U32, P, I, P]),
        "vf_alloc_cuda": (I, [P, U32, P, U64, P, U32, P, I, P]),
        "vf_alloc_packed": (I, [P, U32, P, U64, P, U32, P, P]),
        "vf_reset": (I, [P]),
        "vf_range_table": (I, [P, U32, ctypes.POINTER(ctypes.POINTER(vf_range)), ctypes.POINTER(U32)]),
        "vf_regions": (I, [P, ctypes.POINTER(ctypes.POINTER(vf_region)), ctypes.POINTER(U32)]),
        "vf_type_vptrs": (I, [P, U32, P]),
        "vf_resolve": (I, [P, U32, I, P, U64, P, P]),
        "vf_verify_types": (I, [P, U32, I, P, U64, P, P]),
        "vf_dispatch": (I, [P, I, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_dispatch_cuda": (I, [P, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_dispatch_sharedoa": (I, [P, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_dispatch_coal": (I, [P, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_dispatch_typeptr": (I, [P, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_gol_neighbors": (I, [U32, U32, I, P, P, P]),
        "vf_gol_swap": (I, [P, U64, P, P, P, P, P, P]),
        "vf_gen_swap": (I, [P, U64, P, P, P, P, P, P, P]),
        "vf_checksum_i32": (I, [P, U64, P, P]),
        "vf_launch_count": (U64, []),
        "vf_set_tuning": (I, [ctypes.c_char_p, I]),
        "vf_graph_bfs_init": (I, [U64, P, U32, P, P, U32, P, P, P, P]),
        "vf_iota_u32": (I, [U64, P, P]),
        "vf_fill_f32": (I, [U64, P, ctypes.c_float, P]),
        "vf_ray_render": (I, [P, I, P, U32, U32, U32, U32, U32, P, P, P, P, P]),
        "vf_gol_step": (I, [P, I, U32, U32, I, P, P, P, P, P, P, P]),
        "vf_gol_run": (I, [P, I, U32, U32, I, P, P, P, P, P, P, U32, P, P]),
        "vf_dispatch_host": (I, [P, I, U32, U32, P, U64, P, ctypes.c_size_t, P, U64, P]),
        "vf_dispatch_concord": (I, [P, U32, U32, P, U64, P, ctypes.c_size_t, P]),
        "vf_micro_branch": (I, [U64, U32, I, U64, U32, P, P]),
        "vf_collide_tmp_words": (U64, [U32, U32]),
        "vf_collide_grid": (I, [ctypes.POINTER(collide_grid_args), P]),
        "vf_gen_step": (I, [P, I, U32, U32, I, P, P, P, P, P, P, P, U32, U32, U32, P]),
        "vf_gen_step_rows": (I, [P, I, U32, U32, I, U32, U32, P, P, P, P, P, P, P, U32, U32, U32, P]),
        "vf_collide_pack_near": (I, [U32, U32, P, P, P, P, P, P]),
        "vf_collide_unpack_near": (I, [P, U32, U32, P, U32, U32, U32, P, P, P, P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def app_info(app: int):
    L = lib()
    nt, nm = ctypes.c_uint32(), ctypes.c_uint32()
    sizes = (ctypes.c_uint32 * 128)()
    st = L.vf_app_info(app, ctypes.byref(nt), sizes, ctypes.byref(nm))
    if st:
        raise VFError(st, f"app {app}")
    return int(nt.value), [int(sizes[k]) for k in range(nt.value)], int(nm.value)


def set_tuning(key: str, value: int):
    st = lib().vf_set_tuning(key.encode(), int(value))
    if st:
        raise VFError(st, f"tuning {key}={value}")


def launch_count() -> int:
    return int(lib().vf_launch_count())


def _ptr(t) -> int | None:
    if t is None:
        return None
    return int(t.data_ptr())


def _stream(stream) -> int | None:
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream) if hasattr(s, "cuda_stream") else int(s)


def _args(a) -> tuple:
    if a is None:
        return None, 0
    return ctypes.cast(ctypes.pointer(a), ctypes.c_void_p), ctypes.sizeof(a)


@dataclass
class Range:
    start: int
    end: int
    type_id: int
    app: int
    vptr: int


class Ctx:
    """One vf_ctx (per process and device). Owns every object it allocates."""

    def __init__(self, device: int = 0, init_chunk_objs: int = 4096, reserve_va: bool = True,
                 va_window_bytes: int = 64 << 30, cuda_heap_bytes: int = 8 << 30):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("libvf needs a CUDA device (no CPU fallback)")
        L = lib()
        cfg = vf_config()
        L.vf_config_default(ctypes.byref(cfg))
        cfg.device, cfg.init_chunk_objs, cfg.reserve_va = device, init_chunk_objs, int(reserve_va)
        cfg.va_window_bytes, cfg.cuda_heap_bytes = va_window_bytes, cuda_heap_bytes
        h = ctypes.c_void_p()
        st = L.vf_create(ctypes.byref(cfg), ctypes.byref(h))
        if st:
            raise VFError(st, "vf_create")
        self.h = h
        self.device = device
        self.L = L

    def _check(self, st, what=""):
        if st:
            raise VFError(st, f"{what}: {self.L.vf_last_error(self.h).decode(errors='replace')}")

    def close(self):
        if getattr(self, "h", None):
            self.L.vf_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- allocation ---------------------------------------------------------
    def alloc_typed_batch(self, app, types, ctor_args=None, tag=False, stream=None):
        """types: int32/uint32 CUDA tensor [n]; ctor_args: CUDA tensor [n, ...] (contiguous).
        Returns an int64 CUDA tensor of object pointers (tagged if tag)."""
        import torch
        n = types.numel()
        out = torch.empty(n, dtype=torch.int64, device=types.device)
        ab = 0 if ctor_args is None else ctor_args.element_size() * (ctor_args.numel() // max(n, 1))
        self._check(self.L.vf_alloc_typed_batch(self.h, app, _ptr(types), n, _ptr(ctor_args), ab,
                                                _ptr(out), int(tag), _stream(stream)), "alloc_typed_batch")
        return out

    def alloc_typed(self, app, type_id, count, ctor_args=None, tag=False, stream=None):
        import torch
        out = torch.empty(count, dtype=torch.int64, device=f"cuda:{self.device}")
        ab = 0 if ctor_args is None else ctor_args.element_size() * (ctor_args.numel() // max(count, 1))
        self._check(self.L.vf_alloc_typed(self.h, app, type_id, count, _ptr(ctor_args), ab, _ptr(out),
                                          int(tag), _stream(stream)), "alloc_typed")
        return out

    def alloc_cuda(self, app, types, ctor_args=None, tag=False, stream=None):
        import torch
        n = types.numel()
        out = torch.empty(n, dtype=torch.int64, device=types.device)
        ab = 0 if ctor_args is None else ctor_args.element_size() * (ctor_args.numel() // max(n, 1))
        self._check(self.L.vf_alloc_cuda(self.h, app, _ptr(types), n, _ptr(ctor_args), ab, _ptr(out),
                                         int(tag), _stream(stream)), "alloc_cuda")
        return out

    def alloc_packed(self, app, types, ctor_args=None, stream=None):
        """cuda_packed: placement into one index-ordered slab (dispatch with CUDA)."""
        import torch
        n = types.numel()
        out = torch.empty(n, dtype=torch.int64, device=types.device)
        ab = 0 if ctor_args is None else ctor_args.element_size() * (ctor_args.numel() // max(n, 1))
        self._check(self.L.vf_alloc_packed(self.h, app, _ptr(types), n, _ptr(ctor_args), ab, _ptr(out),
                                           _stream(stream)), "alloc_packed")
        return out

    def alloc_for(self, variant: str, app, types, ctor_args=None, stream=None):
        """The allocation each dispatch variant runs on: device-heap `new` (cuda),
        one index-ordered slab (cuda_packed), or the typed arenas (sharedoa /
        coal / concord untagged, typeptr tagged)."""
        if variant == "cuda":
            return self.alloc_cuda(app, types, ctor_args, stream=stream)
        if variant == "cuda_packed":
            return self.alloc_packed(app, types, ctor_args, stream=stream)
        return self.alloc_typed_batch(app, types, ctor_args, tag=(variant == "typeptr"), stream=stream)

    def reset(self):
        self._check(self.L.vf_reset(self.h), "reset")

    # ---- tables -------------------------------------------------------------
    def range_table(self, app=0xFFFFFFFF):
        p = ctypes.POINTER(vf_range)()
        n = ctypes.c_uint32()
        self._check(self.L.vf_range_table(self.h, app, ctypes.byref(p), ctypes.byref(n)), "range_table")
        return [Range(p[k].start, p[k].end, p[k].type_id, p[k].app, p[k].vptr) for k in range(n.value)]

    def regions(self):
        p = ctypes.POINTER(vf_region)()
        n = ctypes.c_uint32()
        self._check(self.L.vf_regions(self.h, ctypes.byref(p), ctypes.byref(n)), "regions")
        return [dict(start=p[k].start, cap_objs=p[k].cap_objs, used_objs=p[k].used_objs,
                     obj_bytes=p[k].obj_bytes, type_id=p[k].type_id, app=p[k].app)
                for k in range(n.value)]

    def type_vptrs(self, app):
        nt, _, _ = app_info(app)
        buf = (ctypes.c_uint64 * nt)()
        self._check(self.L.vf_type_vptrs(self.h, app, buf), "type_vptrs")
        return [int(x) for x in buf]

    # ---- resolve / verify / dispatch -----------------------------------------
    def resolve(self, app, variant, ptrs, stream=None):
        import torch
        out = torch.empty(ptrs.numel(), dtype=torch.int32, device=ptrs.device)
        self._check(self.L.vf_resolve(self.h, app, variant, _ptr(ptrs), ptrs.numel(), _ptr(out),
                                      _stream(stream)), "resolve")
        return out

    def verify(self, app, variant, ptrs, stream=None) -> int:
        import torch
        m = torch.zeros(1, dtype=torch.int64, device=ptrs.device)
        self._check(self.L.vf_verify_types(self.h, app, variant, _ptr(ptrs), ptrs.numel(), _ptr(m),
                                           _stream(stream)), "verify_types")
        return int(m.item())

    def dispatch(self, variant, app, method, objs, args=None, n=None, stream=None):
        a, ab = _args(args)
        n = objs.numel() if n is None else n
        self._check(self.L.vf_dispatch(self.h, variant, app, method, _ptr(objs), n, a, ab,
                                       _stream(stream)), "dispatch")

    def dispatch_host(self, variant, app, method, objs_host, staging, args=None, chunk=0, stream=None):
        """vf_dispatch_host: objs_host = pinned CPU int64 tensor of object pointers,
        staging = device int64 tensor of the same length (overwritten)."""
        a, ab = _args(args)
        self._check(self.L.vf_dispatch_host(self.h, variant, app, method, objs_host.data_ptr(), objs_host.numel(),
                                            a, ab, _ptr(staging), chunk, _stream(stream)), "dispatch_host")

    def dispatch_raw(self, variant, app, method, objs_ptr: int, n: int, args=None, stream=None):
        """Same as dispatch() with a raw device pointer (hot loops avoid tensor overhead)."""
        a, ab = _args(args)
        return self.L.vf_dispatch(self.h, variant, app, method, objs_ptr, n, a, ab, stream)


def gol_neighbors(W, H, state, nbr, torus=False, stream=None):
    st = lib().vf_gol_neighbors(W, H, int(torus), _ptr(state), _ptr(nbr), _stream(stream))
    if st:
        raise VFError(st, "gol_neighbors")


def gol_swap(ctx: Ctx, prev, nxt, grid, alive, dead, stream=None):
    st = lib().vf_gol_swap(ctx.h, grid.numel(), _ptr(prev), _ptr(nxt), _ptr(grid), _ptr(alive),
                           _ptr(dead), _stream(stream))
    if st:
        raise VFError(st, "gol_swap")


def gen_swap(ctx: Ctx, prev, nxt, grid, dead, alive, dying, stream=None):
    st = lib().vf_gen_swap(ctx.h, grid.numel(), _ptr(prev), _ptr(nxt), _ptr(grid), _ptr(dead),
                           _ptr(alive), _ptr(dying), _stream(stream))
    if st:
        raise VFError(st, "gen_swap")


def gol_step(ctx: Ctx, variant: int, W, H, torus, prev, nxt, nbr, grid, alive, dead, stream=None):
    st = lib().vf_gol_step(ctx.h, variant, W, H, int(torus), _ptr(prev), _ptr(nxt), _ptr(nbr), _ptr(grid),
                           _ptr(alive), _ptr(dead), _stream(stream))
    if st:
        ctx._check(st, "gol_step")


def gol_run(ctx: Ctx, variant: int, W, H, torus, state0, state1, nbr, grid, alive, dead, gens, barrier, stream=None):
    st = lib().vf_gol_run(ctx.h, variant, W, H, int(torus), _ptr(state0), _ptr(state1), _ptr(nbr), _ptr(grid),
                          _ptr(alive), _ptr(dead), gens, _ptr(barrier), _stream(stream))
    if st:
        ctx._check(st, "gol_run")


def gen_step(ctx: Ctx, variant: int, W, H, torus, prev, nxt, nbr, grid, dead, alive, dying, born, survive, C,
             stream=None):
    st = lib().vf_gen_step(ctx.h, variant, W, H, int(torus), _ptr(prev), _ptr(nxt), _ptr(nbr), _ptr(grid),
                           _ptr(dead), _ptr(alive), _ptr(dying), born, survive, C, _stream(stream))
    if st:
        ctx._check(st, "gen_step")


def gen_step_rows(ctx: Ctx, variant: int, W, H, torus, row0, nrows, prev, nxt, nbr, grid, dead, alive, dying,
                  born, survive, C, stream=None):
    st = lib().vf_gen_step_rows(ctx.h, variant, W, H, int(torus), row0, nrows, _ptr(prev), _ptr(nxt), _ptr(nbr),
                                _ptr(grid), _ptr(dead), _ptr(alive), _ptr(dying), born, survive, C,
                                _stream(stream))
    if st:
        ctx._check(st, "gen_step_rows")


def micro_branch(vals, T: int, order: str, seed: int, k: int = 1, stream=None):
    """BRANCH ceiling (vf.h vf_micro_branch): vals[i] += t(i)+1, t from registers."""
    st = lib().vf_micro_branch(vals.numel(), T, ORDERS[order], seed, k, _ptr(vals), _stream(stream))
    if st:
        raise VFError(st, "micro_branch")


def checksum_i32(vals, out, stream=None):
    st = lib().vf_checksum_i32(_ptr(vals), vals.numel(), _ptr(out), _stream(stream))
    if st:
        raise VFError(st, "checksum_i32")


def strip(p: int) -> int:
    return p & ((1 << VA_BITS) - 1)


def as_u64(t) -> np.ndarray:
    """int64 torch tensor of pointers -> numpy uint64 (bit pattern)."""
    return t.cpu().numpy().view(np.uint64)
