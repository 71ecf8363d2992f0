"""ctypes loader for libmario.so (the C-ABI declared in include/mario.h and
include/mario_kernels.h). Argument marshalling only — no computation happens here.
There is no fallback: if the library is missing, importing the product fails loudly."""
from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MARIO_LIB") or os.path.join(_PKG, "libmario.so")

_lib = None

vp, i32, f32, u64, f64 = C.c_void_p, C.c_int32, C.c_float, C.c_uint64, C.c_double

_SIGS = {
    # kernel-level ABI (include/mario_kernels.h)
    "mario_k_gemm_bf16": (i32, [vp, i32, i32, vp, i32, i32, i32, i32, i32, vp, i32, i32, f32,
                                vp, vp, i32, vp, vp, i32, vp]),
    "mario_k_gemm_f32": (i32, [vp, i32, i32, vp, i32, i32, i32, i32, i32, vp, i32, f32, vp,
                               vp, i32, vp, vp, i32, vp]),
    "mario_k_attn_fwd": (i32, [vp, vp, vp, i32, i32, i32, i32, i32, vp]),
    "mario_k_attn_bwd": (i32, [vp, vp, vp, vp, vp, vp, i32, i32, i32, i32, i32, vp]),
    "mario_k_attn_bwd_ws_bytes": (C.c_size_t, [i32, i32, i32, i32]),
    "mario_k_attn_bwd_ws": (i32, [vp, vp, vp, vp, vp, vp, vp, C.c_size_t, i32, i32, i32, i32, vp]),
    "mario_k_norm_fwd": (i32, [vp, vp, vp, vp, vp, i32, i32, f32, i32, i32, vp]),
    "mario_k_norm_bwd": (i32, [vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, C.c_longlong, i32, i32, i32, i32, vp]),
    "mario_k_norm_set_variant": (i32, [i32]),
    "mario_k_softmax_ce": (i32, [vp, vp, i32, i32, i32, i32, f32, vp, vp, i32, vp]),
    "mario_kernel_launches": (C.c_longlong, []),
    "mario_k_gemm_set_variant": (i32, [i32]),
    "mario_k_gemm_set_streamk": (i32, [i32]),
    "mario_k_attn_set_variant": (i32, [i32]),
    "mario_kstats_enable": (i32, [i32]),
    "mario_kstats_read": (i32, [i32, C.POINTER(C.c_double), C.POINTER(C.c_double), C.POINTER(C.c_double),
                                C.POINTER(C.c_longlong)]),
}


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libmario.so not built at {LIB_PATH}: run `python -m "
                               "paper_conf_ppopp_liultj25_b200.build` (no CPU fallback exists)")
        _lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
        for name, (res, args) in _SIGS.items():
            if hasattr(_lib, name):
                fn = getattr(_lib, name)
                fn.restype, fn.argtypes = res, args
    return _lib


def register(name, restype, argtypes):
    _SIGS[name] = (restype, argtypes)
    if _lib is not None and hasattr(_lib, name):
        fn = getattr(_lib, name)
        fn.restype, fn.argtypes = restype, argtypes
