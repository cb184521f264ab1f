"""ctypes loader for the CUDA library ``_flb.so`` (the C ABI of include/flb_paillier.h).

There is no fallback: if the shared library is missing or fails to load, importing the package
raises.  Build it with ``python -c "import __graft_entry__ as g; g.build()"`` (or
``python -m paper_conf_icde_zeng0fcpcwg23_b200.build``).
"""

from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FLB_LIB_PATH") or os.path.join(_HERE, "_flb.so")

FLB_OK = 0
ERRORS = {-1: "FLB_EINVAL", -2: "FLB_ENOMEM", -3: "FLB_ECUDA", -4: "FLB_EKEY", -5: "FLB_EUNSUPPORTED"}


class FlbError(RuntimeError):
    def __init__(self, fn: str, code: int, msg: str):
        super().__init__("%s failed: %s (%d): %s" % (fn, ERRORS.get(code, "?"), code, msg))
        self.code = code


class CodecStruct(ctypes.Structure):
    _fields_ = [("alpha", ctypes.c_double), ("qbits", ctypes.c_uint32), ("pad_bits", ctypes.c_uint32),
                ("slot_bits", ctypes.c_uint32), ("slots", ctypes.c_uint32)]


_P = ctypes.c_void_p
_U32 = ctypes.c_uint32
_U64 = ctypes.c_uint64
_SZ = ctypes.c_size_t

# name -> (restype, argtypes); every symbol include/flb_paillier.h declares
SIGNATURES = {
    "flb_keygen": (ctypes.c_int, [_U32, _U64, ctypes.POINTER(_P), ctypes.POINTER(_P)]),
    "flb_key_from_primes": (ctypes.c_int, [_P, _P, _U32, ctypes.POINTER(_P), ctypes.POINTER(_P)]),
    "flb_key_export": (ctypes.c_int, [_P, _P, _P, _P]),
    "flb_pub_free": (None, [_P]),
    "flb_priv_free": (None, [_P]),
    "flb_key_bits": (_U32, [_P]),
    "flb_pt_words": (_U32, [_P]),
    "flb_ct_words": (_U32, [_P]),
    "flb_slot_capacity": (_U32, [_P, _U32]),
    "flb_encrypt": (ctypes.c_int, [_P, _P, _P, _U64, _U64, _P, _SZ, _P]),
    "flb_encrypt_crt": (ctypes.c_int, [_P, _P, _P, _U64, _U64, _P, _SZ, _P]),
    "flb_decrypt": (ctypes.c_int, [_P, _P, _P, _SZ, _P]),
    "flb_add": (ctypes.c_int, [_P, _P, _P, _P, _SZ, _P]),
    "flb_scalar_mul": (ctypes.c_int, [_P, _P, _P, _U32, _P, _SZ, _P]),
    "flb_reduce_segments": (ctypes.c_int, [_P, _P, _SZ, _P, _SZ, _P, _SZ, _SZ, _P, _P]),
    "flb_multiexp_segments": (ctypes.c_int, [_P, _P, _SZ, _P, _P, _U32, _P, _SZ, _SZ, _P, _P]),
    "flb_pack": (ctypes.c_int, [_P, ctypes.POINTER(CodecStruct), _P, _SZ, _P, _P]),
    "flb_unpack": (ctypes.c_int, [_P, ctypes.POINTER(CodecStruct), _P, _SZ, _P, _U32, _P, _P]),
    "flb_unpack_sums": (ctypes.c_int, [_P, ctypes.POINTER(CodecStruct), _P, _SZ, _P, _P]),
    "flb_debug_mont_mul": (ctypes.c_int, [_P, _P, _P, _P, _SZ, _P]),
    "flb_debug_tc_product": (ctypes.c_int, [_P, _P, _P, _U32, _U32, ctypes.c_int, _P]),
    "flb_mod_create": (ctypes.c_int, [_P, _U32, ctypes.POINTER(_P)]),
    "flb_mod_free": (None, [_P]),
    "flb_mod_words": (_U32, [_P]),
    "flb_mod_mul": (ctypes.c_int, [_P, _P, _P, _P, _SZ, _P]),
    "flb_mod_pow": (ctypes.c_int, [_P, _P, _P, _U32, _P, _SZ, _P]),
    "flb_mod_pow_shared": (ctypes.c_int, [_P, _P, _P, _U32, _P, _SZ, _P]),
    "flb_rsa_keygen": (ctypes.c_int, [_U32, _U64, _U32, _P, _P, _P, _P]),
    "flb_mp_add": (ctypes.c_int, [_P, _P, _P, _P, _U32, _SZ, _P]),
    "flb_mp_sub": (ctypes.c_int, [_P, _P, _P, _P, _U32, _SZ, _P]),
    "flb_mp_mul": (ctypes.c_int, [_P, _P, _P, _U32, _SZ, _P]),
    "flb_mp_divmod": (ctypes.c_int, [_P, _P, _P, _P, _U32, _SZ, _P]),
    "flb_mp_mod": (ctypes.c_int, [_P, _P, _P, _U32, _SZ, _P]),
    "flb_mp_mod_inv": (ctypes.c_int, [_P, _P, _P, _P, _U32, _SZ, _P]),
    "flb_miller_rabin": (ctypes.c_int, [_P, _U32, _P, _U32, _U64, _P, _SZ, _P]),
    "flb_keygen_gpu": (ctypes.c_int, [_U32, _U64, ctypes.POINTER(_P), ctypes.POINTER(_P), _P]),
    "flb_pack_encrypt_host": (ctypes.c_int, [_P, _P, ctypes.POINTER(CodecStruct), _P, _SZ, _U64, _U64, _P]),
    "flb_pack_encrypt_host_multi": (ctypes.c_int, [_P, _P, ctypes.POINTER(CodecStruct), _P, _P, _SZ, _U64, _U64,
                                                    _P]),
    "flb_decrypt_unpack_host": (ctypes.c_int, [_P, _P, ctypes.POINTER(CodecStruct), _P, _SZ, _P, _U32, _P]),
    "flb_reduce_segments_host": (ctypes.c_int, [_P, _P, _SZ, _P, _P, _SZ, _SZ, _P]),
    "flb_op_cost": (ctypes.c_int, [_P, _P, ctypes.c_int, ctypes.POINTER(_U64), ctypes.POINTER(_U64)]),
    "flb_last_error": (ctypes.c_char_p, []),
    "flb_version": (ctypes.c_char_p, []),
}


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    if not os.path.exists(path):
        raise ImportError("CUDA library %s is not built; run __graft_entry__.build()" % path)
    lib = ctypes.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


LIB = load()


def check(fn: str, rc: int) -> None:
    if rc != FLB_OK:
        raise FlbError(fn, rc, LIB.flb_last_error().decode())
