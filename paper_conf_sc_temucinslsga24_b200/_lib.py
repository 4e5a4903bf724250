"""ctypes loader for the in-tree C-ABI libraries (argument marshalling only).

``libpc.so``     the product: include/pc.h (host ABI) + device engines.
``libpcapps.so`` producer / application kernels compiled against
                 include/pc_device.cuh (what a user's kernel looks like).

There is no fallback: if the shared objects are missing this raises.  Build
them with ``python -c "import __graft_entry__ as g; g.build()"`` (or ``make -C
paper_conf_sc_temucinslsga24_b200/csrc``).
"""
from __future__ import annotations

import ctypes as C
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
LIBPC = os.environ.get("PC_LIB") or os.path.join(_HERE, "libpc.so")
LIBAPPS = os.environ.get("PC_APPS_LIB") or os.path.join(_HERE, "libpcapps.so")
INCLUDE = os.path.join(os.path.dirname(_HERE), "include")

P = C.c_void_p
I32 = C.c_int
I64 = C.c_int64
SZ = C.c_size_t
PI32 = C.POINTER(C.c_int32)
PI64 = C.POINTER(C.c_int64)

AGFN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)

# name -> (restype, argtypes)
_PC_PROTOS = {
    "pc_comm_create": (I32, [I32, I32, I32, P, P, C.POINTER(P)]),
    "pc_comm_destroy": (I32, [P]),
    "pc_comm_rank": (I32, [P, PI32]),
    "pc_comm_size": (I32, [P, PI32]),
    "pc_comm_engine_warps": (I32, [P, PI32]),
    "pc_comm_overlap_warps": (I32, [P, PI32]),
    "pc_local_group_create": (I32, [I32, C.POINTER(P)]),
    "pc_local_group_destroy": (I32, [P]),
    "pc_local_group_ctx": (P, [P, I32]),
    "pc_local_allgather": (I32, [P, SZ, P, P]),
    "pc_psend_init": (I32, [P, I32, SZ, I32, I32, I32, P, C.POINTER(P)]),
    "pc_precv_init": (I32, [P, I32, SZ, I32, I32, I32, P, C.POINTER(P)]),
    "pc_pallreduce_init": (I32, [P, P, I32, SZ, I32, I32, I32, P, C.POINTER(P)]),
    "pc_preduce_scatter_init": (I32, [P, P, I32, SZ, I32, I32, P, C.POINTER(P)]),
    "pc_pallgather_init": (I32, [P, P, I32, SZ, I32, P, C.POINTER(P)]),
    "pc_pbcast_init": (I32, [P, I32, SZ, I32, I32, P, C.POINTER(P)]),
    "pc_start": (I32, [P, P]),
    "pc_startall": (I32, [I32, P, P]),
    "pc_epoch_all": (I32, [I32, P, I32, P]),
    "pc_pbuf_prepare_all": (I32, [I32, P, P]),
    "pc_pbuf_prepare": (I32, [P, P]),
    "pc_prequest_create": (I32, [P, I32, I32, I32, P]),
    "pc_prequest_free": (I32, [P]),
    "pc_prequest_size": (SZ, []),
    "pc_parrived": (I32, [P, I32, PI32]),
    "pc_test": (I32, [P, PI32]),
    "pc_wait": (I32, [P]),
    "pc_wait_on_stream": (I32, [P, P]),
    "pc_waitall_on_stream": (I32, [I32, P, P]),
    "pc_pready": (I32, [I32, P, P]),
    "pc_pready_range": (I32, [I32, I32, P, P]),
    "pc_preadyall": (I32, [I32, P, P]),
    "pc_request_free": (I32, [C.POINTER(P)]),
    "pc_schedule_ring": (I32, [I32, I32, PI32]),
    "pc_schedule_rd": (I32, [I32, I32, PI32]),
    "pc_chunk_bounds": (I32, [I64, I32, PI64]),
    "pc_request_info": (I32, [P, PI32, PI32, PI64, PI32]),
    "pc_request_match": (I32, [P, PI32, PI32]),
    "pc_request_error": (I32, [P, PI32, PI32]),
    "pc_request_words": (I32, [P, I32, I32, I32, P]),
    "pc_request_set_timing": (I32, [P, I32]),
    "pc_request_set_overlap": (I32, [P, I32]),
    "pc_request_peer_buffer": (I32, [P, I32, C.POINTER(C.c_void_p)]),
    "pc_request_engine_times": (I32, [P, P, I32]),
    "pc_launch_count": (C.c_uint64, []),
    "pc_strerror": (C.c_char_p, [I32]),
    "pc_version": (C.c_char_p, []),
}

_APP_PROTOS = {
    "pcapp_vecadd": (I32, [P, P, P, I64, I32, P, P]),
    "pcapp_vecadd_persistent": (I32, [P, P, P, I64, I32, P, P]),
    "pcapp_produce_put": (I32, [P, P, I32, I64, I32, I32, I32, P, P]),
    "pcapp_pready_cost": (I32, [P, P, P, I32, I32, P, P, P]),
    "pcapp_produce": (I32, [P, P, I32, I64, I32, I32, I32, P, P]),
    "pcapp_bce_grad": (I32, [P, P, P, I32, I64, C.c_float, I32, I32, P, P]),
    "pcapp_bce_grad_multi": (I32, [I32, P, P, P, I32, I64, C.c_float, I32, P, I32, P]),
    "pcapp_check_recv": (I32, [P, P, P, I32, I64, I32, P, P]),
    "pcapp_pingpong": (I32, [P, P, I32, I32, I32, P, P]),
    "pcapp_bare_pingpong": (I32, [P, P, I32, I32, C.c_uint32, P, P]),
    "pcapp_pingpong_pair": (I32, [P, P, P, P, I32, I32, P, P, P]),
    "pcapp_bare_pingpong_pair": (I32, [P, P, I32, C.c_uint32, P, I32, P]),
    "pcapp_prequest_size": (SZ, []),
    "pcapp_overlap_probe": (I32, [C.POINTER(P), I32, I32, C.c_uint32, P, P]),
    "pcapp_peer_copy": (I32, [I32, C.POINTER(P), C.POINTER(P), C.c_uint64, I32, P]),
    "pcapp_memcpy_async": (I32, [P, P, C.c_uint64, P]),
    "pcapp_flag_variant": (I32, [P, P, I32, I32, C.c_uint32, P, P]),
    "pcapp_lat_probe_pair": (I32, [P, P, P, P, I32, I32, P, P]),
    "pcapp_jacobi_rank_size": (SZ, []),
    "pcapp_jacobi_launch": (I32, [P, P, I32, I32, I32, I32, P]),
    "pcapp_jacobi_describe": (I32, [P, P, P, I32, I32, I32, I32, I32, I32, P, P, P, P, P]),
    "pcapp_jacobi_set_traditional": (I32, [P, I32]),
    "pcapp_jacobi_launch2": (I32, [P, P, I32, I32, I32, I32, I32, I32, I32, P]),
    "pcapp_jacobi_describe2": (I32, [P, P, P, I32, I32, I32, I32, I32, I32, P, P, P, P, P, I32, I32]),
}

_pc = None
_apps = None


class LibraryMissing(RuntimeError):
    pass


def _load(path, protos):
    if not os.path.exists(path):
        raise LibraryMissing(f"{path} is not built; run __graft_entry__.build() (no CPU fallback exists)")
    lib = C.CDLL(path, mode=C.RTLD_GLOBAL)
    for name, (res, args) in protos.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


def pc():
    global _pc
    if _pc is None:
        _pc = _load(LIBPC, _PC_PROTOS)
    return _pc


def apps():
    global _apps
    if _apps is None:
        pc()
        _apps = _load(LIBAPPS, _APP_PROTOS)
        assert _apps.pcapp_prequest_size() == pc().pc_prequest_size(), "pc_prequest_t layout mismatch"
    return _apps


def header_symbols(header: str = "pc.h") -> list[str]:
    """Every function declared in include/<header> (for the export check)."""
    text = open(os.path.join(INCLUDE, header)).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(pc_[a-z0-9_]+)\s*\(", text)) - {"pc_allgather_fn"})
