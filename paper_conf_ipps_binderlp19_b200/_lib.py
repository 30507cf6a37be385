"""ctypes loader for libsnp.so — the C ABI declared in include/snp.h.

No fallback: if the shared object is missing or fails to load, every call
raises.  (Build it with ``python -m paper_conf_ipps_binderlp19_b200.build`` or
``__graft_entry__.build()``.)
"""
from __future__ import annotations

import ctypes
import os
import threading

LIB_PATH = os.environ.get("SNP_LIB_PATH") or os.path.join(os.path.dirname(os.path.abspath(__file__)), "libsnp.so")

# Every symbol include/snp.h declares: name -> (restype, argtypes)
_i64, _int, _sz, _p = ctypes.c_int64, ctypes.c_int, ctypes.c_size_t, ctypes.c_void_p
SIGNATURES = {
    "snp_words": (_i64, [_i64]),
    "snp_ld_workspace_bytes": (_sz, [_i64, _i64, _i64]),
    "snp_fastid_workspace_bytes": (_sz, [_i64, _i64, _i64, _int]),
    "snp_pack": (_int, [_p, _i64, _i64, _i64, _p, _i64, _p]),
    "snp_row_popc": (_int, [_p, _i64, _i64, _i64, _p, _p]),
    "snp_pack_popc": (_int, [_p, _i64, _i64, _i64, _p, _i64, _p, _p]),
    "snp_ld_counts": (_int, [_p, _i64, _i64, _p, _i64, _i64, _i64, _p, _i64, _int, _p, _sz, _p]),
    "snp_ld_r2": (_int, [_p, _i64, _i64, _p, _p, _i64, _i64, _p, _i64, _p, _p, _p, _i64, _p, _sz, _p]),
    "snp_fastid": (_int, [_p, _i64, _i64, _p, _p, _i64, _i64, _p, _i64, _int, _p, _i64, _int, _p, _sz, _p]),
    "snp_fastid_best": (_int, [_p, _i64, _i64, _i64, _i64, _p, _p, _p]),
    "snp_fastid_search_workspace_bytes": (_sz, [_i64, _i64, _i64, _int]),
    "snp_fastid_search": (_int, [_p, _i64, _i64, _p, _i64, _i64, _p, _i64, _int, _p, _p, _i64, _p, _p, _i64,
                                 _p, _sz, _p]),
    "snp_shard_plan": (_int, [_i64, _int, _i64, _p]),
    "snp_fastid_threshold_workspace_bytes": (_sz, [_i64, _i64, _i64, _int]),
    "snp_fastid_threshold": (_int, [_p, _i64, _i64, _p, _i64, _i64, _p, _i64, _int, ctypes.c_uint32, _i64, _p, _i64,
                                    _p, _p, _sz, _p]),
    "snp_shard_plan_sym": (_int, [_i64, _int, _p]),
    "snp_sym_tiles": (_i64, [_i64]),
    "snp_ld_sym_workspace_bytes": (_sz, [_i64, _i64]),
    "snp_ld_sym": (_int, [_p, _i64, _i64, _p, _i64, _i64, _i64, _p, _p, _p, _p, _sz, _p]),
    "snp_sym_unpack": (_int, [_p, _i64, _i64, _i64, _p, _i64, _p]),
    "snp_set_variant": (_int, [_int]),
    "snp_last_variant": (_int, []),
    "snp_launch_count": (_i64, []),
    "snp_last_kernel": (_int, []),
    "snp_status_string": (ctypes.c_char_p, [_int]),
    "snp_last_cuda_error": (ctypes.c_char_p, []),
}

_lock = threading.Lock()
_lib = None


class SnpError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str = ""):
        self.status = status
        msg = f"{where}: {status_string(status) if _lib else status}"
        if detail:
            msg += f" ({detail})"
        super().__init__(msg)


def lib():
    global _lib
    if _lib is None:
        with _lock:
            if _lib is None:
                if not os.path.exists(LIB_PATH):
                    raise RuntimeError(
                        f"libsnp.so not found at {LIB_PATH}: the CUDA library must be built "
                        "(python -m paper_conf_ipps_binderlp19_b200.build); there is no fallback")
                L = ctypes.CDLL(LIB_PATH)
                for name, (res, args) in SIGNATURES.items():
                    f = getattr(L, name)
                    f.restype = res
                    f.argtypes = args
                _lib = L
    return _lib


def status_string(s: int) -> str:
    return lib().snp_status_string(s).decode()


def check(status: int, where: str):
    if status != 0:
        detail = lib().snp_last_cuda_error().decode() if status == 8 else ""
        raise SnpError(status, where, detail)
