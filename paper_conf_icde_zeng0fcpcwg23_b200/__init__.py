"""flb-b200: batched Paillier homomorphic encryption for NVIDIA B200 (FLBooster hot path).

Thin Python binding over the C ABI in ``include/flb_paillier.h`` (argument marshalling only —
every step of the path runs in the CUDA kernels of ``csrc/``; there is no CPU fallback).
PyTorch provides device memory and streams: batches are CUDA ``torch.int32`` tensors of shape
``[count, words]`` holding little-endian 32-bit limbs, launched on
``torch.cuda.current_stream()``.

Paper: Zeng et al., "FLBooster", ICDE 2023 (``PAPER L<n>`` = /root/reference/PAPER.md line n).
"""

from __future__ import annotations

import ctypes
from typing import Optional, Tuple, Union

import torch

from . import _lib
from ._lib import LIB, FlbError, check

__all__ = [
    "PublicKey", "PrivateKey", "keygen", "key_from_primes", "encrypt", "encrypt_crt", "decrypt", "add",
    "scalar_mul", "reduce_segments", "multiexp_segments", "pack", "unpack", "unpack_sums", "debug_mont_mul",
    "Codec", "FlbError", "library_path", "op_cost", "keygen_gpu", "miller_rabin", "Modulus", "rsa_keygen", "pack_encrypt_host", "decrypt_unpack_host",
    "reduce_segments_host", "pack_encrypt_host_multi", "mp_add", "mp_sub", "mp_mul", "mp_divmod", "mp_mod",
    "mp_mod_inv",
]

library_path = _lib.LIB_PATH


def _stream(stream: Optional[torch.cuda.Stream] = None) -> ctypes.c_void_p:
    """The launch stream: `stream`, else the current stream of the CURRENT device — callers run
    inside ``_on(tensor)``, which makes the tensors' device current (the library launches on and
    uploads key constants to the current device)."""
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _on(t: torch.Tensor):
    """Make t's device the current CUDA device for the duration of a library call."""
    return torch.cuda.device(t.device)


def _ptr(t: Optional[torch.Tensor]) -> Optional[int]:
    return None if t is None else t.data_ptr()


def _check_batch(t: torch.Tensor, words: int, name: str, rows: Optional[int] = None,
                 like: Optional[torch.Tensor] = None) -> int:
    """Validate a [count, words] limb batch; ``rows``: required row count (an output buffer or a
    second operand); ``like``: must live on the same device."""
    if not t.is_cuda:
        raise ValueError("%s must be a CUDA tensor" % name)
    if t.dtype not in (torch.int32, torch.uint32):
        raise ValueError("%s must be int32/uint32 limbs" % name)
    if t.dim() != 2 or t.shape[1] != words or not t.is_contiguous():
        raise ValueError("%s must be a contiguous [count, %d] tensor, got %s" % (name, words, tuple(t.shape)))
    if t.data_ptr() % 16:
        raise ValueError("%s must be 16-byte aligned" % name)
    if rows is not None and t.shape[0] != rows:
        raise ValueError("%s must have %d rows, got %d" % (name, rows, t.shape[0]))
    if like is not None and t.device != like.device:
        raise ValueError("%s is on %s, expected %s" % (name, t.device, like.device))
    return t.shape[0]


def _check_vec(t: torch.Tensor, dtypes, name: str, min_len: int, like: torch.Tensor) -> None:
    if not t.is_cuda or t.dtype not in dtypes or t.dim() != 1 or not t.is_contiguous():
        raise ValueError("%s must be a contiguous CUDA %s vector" % (name, "/".join(str(d) for d in dtypes)))
    if t.shape[0] < min_len:
        raise ValueError("%s must have at least %d entries, got %d" % (name, min_len, t.shape[0]))
    if t.device != like.device:
        raise ValueError("%s is on %s, expected %s" % (name, t.device, like.device))


def _limbs_of(x: int, words: int):
    arr = (ctypes.c_uint32 * words)()
    for i in range(words):
        arr[i] = (x >> (32 * i)) & 0xFFFFFFFF
    return arr


class PublicKey:
    """Public key (n, g = n + 1): PAPER L89."""

    def __init__(self, handle: ctypes.c_void_p):
        self._h = handle
        self.bits = LIB.flb_key_bits(handle)
        self.pt_words = LIB.flb_pt_words(handle)
        self.ct_words = LIB.flb_ct_words(handle)

    @property
    def handle(self):
        return self._h

    def slot_capacity(self, slot_bits: int) -> int:
        return LIB.flb_slot_capacity(self._h, slot_bits)

    def __del__(self, _free=LIB.flb_pub_free):
        h, self._h = getattr(self, "_h", None), None
        if h:
            _free(h)


class PrivateKey:
    """Private key (p, q): PAPER L89."""

    def __init__(self, handle: ctypes.c_void_p, pub: PublicKey):
        self._h = handle
        self.pub = pub

    @property
    def handle(self):
        return self._h

    def export(self) -> Tuple[int, int, int]:
        """(p, q, n) as Python ints, p > q."""
        half = self.pub.pt_words // 2
        p = (ctypes.c_uint32 * half)()
        q = (ctypes.c_uint32 * half)()
        n = (ctypes.c_uint32 * self.pub.pt_words)()
        check("flb_key_export", LIB.flb_key_export(self._h, p, q, n))
        to_int = lambda a: sum(int(w) << (32 * i) for i, w in enumerate(a))
        return to_int(p), to_int(q), to_int(n)

    def __del__(self, _free=LIB.flb_priv_free):
        h, self._h = getattr(self, "_h", None), None
        if h:
            _free(h)


def keygen(key_bits: int, seed: int) -> Tuple[PublicKey, PrivateKey]:
    """Paillier::key_gen: deterministic host key generation."""
    pub, priv = ctypes.c_void_p(), ctypes.c_void_p()
    check("flb_keygen", LIB.flb_keygen(key_bits, seed & 0xFFFFFFFFFFFFFFFF, ctypes.byref(pub), ctypes.byref(priv)))
    P = PublicKey(pub)
    return P, PrivateKey(priv, P)


def keygen_gpu(key_bits: int, seed: int, stream=None) -> Tuple[PublicKey, PrivateKey]:
    """Paillier::key_gen on the device: Philox candidates, sieve and Miller–Rabin kernels."""
    pub, priv = ctypes.c_void_p(), ctypes.c_void_p()
    check("flb_keygen_gpu", LIB.flb_keygen_gpu(key_bits, seed & 0xFFFFFFFFFFFFFFFF, ctypes.byref(pub), ctypes.byref(priv),
                                               _stream(stream)))
    P = PublicKey(pub)
    return P, PrivateKey(priv, P)


def miller_rabin(cand: torch.Tensor, rounds: int, mont_bases: Optional[torch.Tensor] = None, seed: int = 0,
                 out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """Miller–Rabin verdicts (int32 [count], 1 = probable prime) for candidates [count, words]."""
    words = cand.shape[1]
    M = _check_batch(cand, words, "cand")
    if mont_bases is not None:
        _check_batch(mont_bases, words, "mont_bases", rows=M * rounds, like=cand)
    if out is None:
        out = torch.empty((M,), dtype=torch.int32, device=cand.device)
    _check_vec(out, (torch.int32, torch.uint32), "out", M, cand)
    with _on(cand):
        check("flb_miller_rabin", LIB.flb_miller_rabin(_ptr(cand), words, _ptr(mont_bases), rounds,
                                                       seed & 0xFFFFFFFFFFFFFFFF, _ptr(out), M, _stream(stream)))
    return out


def key_from_primes(p: int, q: int) -> Tuple[PublicKey, PrivateKey]:
    """Import a key from its primes (e.g. the oracle's, for parity tests)."""
    words = max((max(p, q).bit_length() + 31) // 32, 1)
    pub, priv = ctypes.c_void_p(), ctypes.c_void_p()
    check("flb_key_from_primes", LIB.flb_key_from_primes(_limbs_of(p, words), _limbs_of(q, words), words,
                                                         ctypes.byref(pub), ctypes.byref(priv)))
    P = PublicKey(pub)
    return P, PrivateKey(priv, P)


def encrypt(pub: PublicKey, m: torch.Tensor, r: Optional[torch.Tensor] = None, seed: int = 0, ctr0: int = 0,
            out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """Paillier::encrypt (Eq. 3): c = (1 + m n) r^n mod n^2; r = Philox(seed, ctr0 + i) if None."""
    M = _check_batch(m, pub.pt_words, "m")
    if r is not None:
        _check_batch(r, pub.pt_words, "r", rows=M, like=m)
    if out is None:
        out = torch.empty((M, pub.ct_words), dtype=torch.int32, device=m.device)
    _check_batch(out, pub.ct_words, "out", rows=M, like=m)
    with _on(m):
        check("flb_encrypt", LIB.flb_encrypt(pub.handle, _ptr(m), _ptr(r), seed & 0xFFFFFFFFFFFFFFFF, ctr0, _ptr(out),
                                             M, _stream(stream)))
    return out


def encrypt_crt(priv: PrivateKey, m: torch.Tensor, r: Optional[torch.Tensor] = None, seed: int = 0, ctr0: int = 0,
                out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """Key-holder encryption: the same ciphertexts as ``encrypt`` via CRT over p^2, q^2 (~2x fewer limb products)."""
    pub = priv.pub
    M = _check_batch(m, pub.pt_words, "m")
    if r is not None:
        _check_batch(r, pub.pt_words, "r", rows=M, like=m)
    if out is None:
        out = torch.empty((M, pub.ct_words), dtype=torch.int32, device=m.device)
    _check_batch(out, pub.ct_words, "out", rows=M, like=m)
    with _on(m):
        check("flb_encrypt_crt", LIB.flb_encrypt_crt(priv.handle, _ptr(m), _ptr(r), seed & 0xFFFFFFFFFFFFFFFF, ctr0,
                                                     _ptr(out), M, _stream(stream)))
    return out


def decrypt(priv: PrivateKey, c: torch.Tensor, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """Paillier::decrypt (Eq. 4) by CRT."""
    pub = priv.pub
    M = _check_batch(c, pub.ct_words, "c")
    if out is None:
        out = torch.empty((M, pub.pt_words), dtype=torch.int32, device=c.device)
    _check_batch(out, pub.pt_words, "out", rows=M, like=c)
    with _on(c):
        check("flb_decrypt", LIB.flb_decrypt(priv.handle, _ptr(c), _ptr(out), M, _stream(stream)))
    return out


def add(pub: PublicKey, c1: torch.Tensor, c2: torch.Tensor, out: Optional[torch.Tensor] = None,
        stream=None) -> torch.Tensor:
    """Paillier::add (Eq. 5): c1 c2 mod n^2."""
    M = _check_batch(c1, pub.ct_words, "c1")
    _check_batch(c2, pub.ct_words, "c2", rows=M, like=c1)
    if out is None:
        out = torch.empty_like(c1)
    _check_batch(out, pub.ct_words, "out", rows=M, like=c1)
    with _on(c1):
        check("flb_add", LIB.flb_add(pub.handle, _ptr(c1), _ptr(c2), _ptr(out), M, _stream(stream)))
    return out


def scalar_mul(pub: PublicKey, c: torch.Tensor, e: torch.Tensor, out: Optional[torch.Tensor] = None,
               stream=None) -> torch.Tensor:
    """c^e mod n^2 = E(e m) (mod_pow); e: [count, e_words] unsigned limbs."""
    M = _check_batch(c, pub.ct_words, "c")
    if e.dim() != 2:
        raise ValueError("e must be [count, e_words]")
    _check_batch(e, e.shape[1], "e", rows=M, like=c)
    if out is None:
        out = torch.empty_like(c)
    _check_batch(out, pub.ct_words, "out", rows=M, like=c)
    with _on(c):
        check("flb_scalar_mul", LIB.flb_scalar_mul(pub.handle, _ptr(c), _ptr(e), e.shape[1], _ptr(out), M,
                                                   _stream(stream)))
    return out


def reduce_segments(pub: PublicKey, c: torch.Tensor, offsets: torch.Tensor, idx: Optional[torch.Tensor] = None,
                    max_segment_len: int = 0, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """out[j] = prod_{t in [off[j], off[j+1])} c[idx[t]] mod n^2 (empty = 1)."""
    L = _check_batch(c, pub.ct_words, "c")
    _check_vec(offsets, (torch.int64,), "offsets", 1, c)
    S = offsets.shape[0] - 1
    if idx is not None:
        _check_vec(idx, (torch.int64,), "idx", 0, c)
    if out is None:
        out = torch.empty((S, pub.ct_words), dtype=torch.int32, device=c.device)
    _check_batch(out, pub.ct_words, "out", rows=S, like=c)
    nent = idx.shape[0] if idx is not None else L
    with _on(c):
        check("flb_reduce_segments", LIB.flb_reduce_segments(pub.handle, _ptr(c), L, _ptr(idx), nent, _ptr(offsets),
                                                             S, max_segment_len, _ptr(out), _stream(stream)))
    return out


def multiexp_segments(pub: PublicKey, c: torch.Tensor, e: torch.Tensor, offsets: torch.Tensor,
                      idx: Optional[torch.Tensor] = None, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """out[j] = prod_{t in seg j} c[idx[t]]^(e[t]) mod n^2 (per-entry exponents e [entries, e_words])."""
    L = _check_batch(c, pub.ct_words, "c")
    _check_vec(offsets, (torch.int64,), "offsets", 1, c)
    S = offsets.shape[0] - 1
    if e.dim() != 2:
        raise ValueError("e must be [entries, e_words]")
    nent = e.shape[0]
    _check_batch(e, e.shape[1], "e", like=c)
    if idx is not None:
        _check_vec(idx, (torch.int64,), "idx", nent, c)
    elif nent > L:
        raise ValueError("without idx, e must have at most as many rows as c")
    if out is None:
        out = torch.empty((S, pub.ct_words), dtype=torch.int32, device=c.device)
    _check_batch(out, pub.ct_words, "out", rows=S, like=c)
    with _on(c):
        check("flb_multiexp_segments", LIB.flb_multiexp_segments(pub.handle, _ptr(c), L, _ptr(idx), _ptr(e),
                                                                 e.shape[1], _ptr(offsets), S, nent, _ptr(out),
                                                                 _stream(stream)))
    return out


class Codec:
    """Encoding-quantisation / batch-compression parameters (PAPER §IV-B, §IV-C)."""

    def __init__(self, alpha: float, qbits: int, pad_bits: int, slots: int):
        self.alpha, self.qbits, self.pad_bits, self.slots = float(alpha), int(qbits), int(pad_bits), int(slots)
        self.slot_bits = self.qbits + self.pad_bits

    def struct(self) -> _lib.CodecStruct:
        return _lib.CodecStruct(self.alpha, self.qbits, self.pad_bits, self.slot_bits, self.slots)

    def num_plaintexts(self, n_values: int) -> int:
        return -(-n_values // self.slots)


def pack(pub: PublicKey, codec: Codec, x: torch.Tensor, out: Optional[torch.Tensor] = None,
         stream=None) -> torch.Tensor:
    """Quantise + pack float32 values into plaintexts (Eq. 6–9)."""
    if not x.is_cuda or x.dtype != torch.float32 or x.dim() != 1 or not x.is_contiguous():
        raise ValueError("x must be a contiguous CUDA float32 vector")
    M = codec.num_plaintexts(x.shape[0])
    if out is None:
        out = torch.empty((M, pub.pt_words), dtype=torch.int32, device=x.device)
    _check_batch(out, pub.pt_words, "out", rows=M, like=x)
    cs = codec.struct()
    with _on(x):
        check("flb_pack", LIB.flb_pack(pub.handle, ctypes.byref(cs), _ptr(x), x.shape[0], _ptr(out),
                                       _stream(stream)))
    return out


def unpack(pub: PublicKey, codec: Codec, pt: torch.Tensor, n_values: int,
           summands: Union[int, torch.Tensor] = 1, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
    """Unpack + dequantise: x = Sum/sigma - cnt*alpha (float64 -> float32)."""
    npt = codec.num_plaintexts(n_values)
    if _check_batch(pt, pub.pt_words, "pt") < npt:
        raise ValueError("pt must have at least %d rows for %d values" % (npt, n_values))
    if out is None:
        out = torch.empty((n_values,), dtype=torch.float32, device=pt.device)
    _check_vec(out, (torch.float32,), "out", n_values, pt)
    cs = codec.struct()
    if isinstance(summands, torch.Tensor):
        _check_vec(summands, (torch.int32, torch.uint32), "summands", npt, pt)
        sp, ss = _ptr(summands), 0
    else:
        sp, ss = None, int(summands)
    with _on(pt):
        check("flb_unpack", LIB.flb_unpack(pub.handle, ctypes.byref(cs), _ptr(pt), n_values, sp, ss, _ptr(out),
                                           _stream(stream)))
    return out


def unpack_sums(pub: PublicKey, codec: Codec, pt: torch.Tensor, n_values: int, out: Optional[torch.Tensor] = None,
                stream=None) -> torch.Tensor:
    """The exact slot integers (int64 view of uint64)."""
    npt = codec.num_plaintexts(n_values)
    if _check_batch(pt, pub.pt_words, "pt") < npt:
        raise ValueError("pt must have at least %d rows for %d values" % (npt, n_values))
    if out is None:
        out = torch.empty((n_values,), dtype=torch.int64, device=pt.device)
    _check_vec(out, (torch.int64,), "out", n_values, pt)
    cs = codec.struct()
    with _on(pt):
        check("flb_unpack_sums", LIB.flb_unpack_sums(pub.handle, ctypes.byref(cs), _ptr(pt), n_values, _ptr(out),
                                                     _stream(stream)))
    return out


# ----------------------------------------------------------------------------- Table I generic API, RSA
class Modulus:
    """An odd modulus for Table I's mod_mul / mod_pow and RSA (L247–L251)."""

    def __init__(self, n: int):
        words = max(1, (n.bit_length() + 31) // 32)
        h = ctypes.c_void_p()
        check("flb_mod_create", LIB.flb_mod_create(_limbs_of(n, words), words, ctypes.byref(h)))
        self._h, self.n = h, n
        self.words = LIB.flb_mod_words(h)

    def __del__(self, _free=LIB.flb_mod_free):
        h, self._h = getattr(self, "_h", None), None
        if h:
            _free(h)

    def mul(self, a: torch.Tensor, b: torch.Tensor, out=None, stream=None) -> torch.Tensor:
        M = _check_batch(a, self.words, "a")
        _check_batch(b, self.words, "b", rows=M, like=a)
        out = torch.empty_like(a) if out is None else out
        _check_batch(out, self.words, "out", rows=M, like=a)
        with _on(a):
            check("flb_mod_mul", LIB.flb_mod_mul(self._h, _ptr(a), _ptr(b), _ptr(out), M, _stream(stream)))
        return out

    def pow(self, base: torch.Tensor, e: torch.Tensor, out=None, stream=None) -> torch.Tensor:
        """Per-element exponents e [count, e_words] (device)."""
        M = _check_batch(base, self.words, "base")
        if e.dim() != 2:
            raise ValueError("e must be [count, e_words]")
        _check_batch(e, e.shape[1], "e", rows=M, like=base)
        out = torch.empty_like(base) if out is None else out
        _check_batch(out, self.words, "out", rows=M, like=base)
        with _on(base):
            check("flb_mod_pow", LIB.flb_mod_pow(self._h, _ptr(base), _ptr(e), e.shape[1], _ptr(out), M,
                                                 _stream(stream)))
        return out

    def pow_shared(self, base: torch.Tensor, e: int, out=None, stream=None) -> torch.Tensor:
        """One exponent (a Python int) for the whole batch."""
        M = _check_batch(base, self.words, "base")
        ew = max(1, (e.bit_length() + 31) // 32)
        out = torch.empty_like(base) if out is None else out
        _check_batch(out, self.words, "out", rows=M, like=base)
        with _on(base):
            check("flb_mod_pow_shared", LIB.flb_mod_pow_shared(self._h, _ptr(base), _limbs_of(e, ew), ew, _ptr(out),
                                                               M, _stream(stream)))
        return out


def rsa_keygen(key_bits: int, seed: int, e: int = 65537) -> Tuple[int, int, int, int, int]:
    """RSA::key_gen: (n, e, d, p, q) as Python ints (host C++ keygen)."""
    w = key_bits // 32
    n, d = (ctypes.c_uint32 * w)(), (ctypes.c_uint32 * w)()
    p, q = (ctypes.c_uint32 * (w // 2))(), (ctypes.c_uint32 * (w // 2))()
    check("flb_rsa_keygen", LIB.flb_rsa_keygen(key_bits, seed & 0xFFFFFFFFFFFFFFFF, e, n, d, p, q))
    to_int = lambda a: sum(int(x) << (32 * i) for i, x in enumerate(a))
    return to_int(n), e, to_int(d), to_int(p), to_int(q)


# ----------------------------------------------------------------------------- Table I fundamentals
def _mp_operands(a: torch.Tensor, b: torch.Tensor, name_a: str = "a", name_b: str = "b") -> Tuple[int, int]:
    if a.dim() != 2:
        raise ValueError("%s must be [count, words]" % name_a)
    words = a.shape[1]
    M = _check_batch(a, words, name_a)
    _check_batch(b, words, name_b, rows=M, like=a)
    return M, words


def _mp_flag(flag, M, like):
    if flag is None:
        return None
    _check_vec(flag, (torch.int32, torch.uint32), "flag", M, like)
    return flag


def mp_add(a: torch.Tensor, b: torch.Tensor, out=None, carry=None, stream=None) -> torch.Tensor:
    """Table I add: (a + b) mod 2^(32 words) per row; ``carry`` (int32 [count]) receives the
    carry out."""
    M, w = _mp_operands(a, b)
    out = torch.empty_like(a) if out is None else out
    _check_batch(out, w, "out", rows=M, like=a)
    with _on(a):
        check("flb_mp_add", LIB.flb_mp_add(_ptr(a), _ptr(b), _ptr(out), _ptr(_mp_flag(carry, M, a)), w, M,
                                           _stream(stream)))
    return out


def mp_sub(a: torch.Tensor, b: torch.Tensor, out=None, borrow=None, stream=None) -> torch.Tensor:
    """Table I sub: (a - b) mod 2^(32 words); ``borrow`` = 1 where a < b."""
    M, w = _mp_operands(a, b)
    out = torch.empty_like(a) if out is None else out
    _check_batch(out, w, "out", rows=M, like=a)
    with _on(a):
        check("flb_mp_sub", LIB.flb_mp_sub(_ptr(a), _ptr(b), _ptr(out), _ptr(_mp_flag(borrow, M, a)), w, M,
                                           _stream(stream)))
    return out


def mp_mul(a: torch.Tensor, b: torch.Tensor, out=None, stream=None) -> torch.Tensor:
    """Table I mul: the full product a b, [count, 2 words]."""
    M, w = _mp_operands(a, b)
    out = torch.empty((M, 2 * w), dtype=torch.int32, device=a.device) if out is None else out
    _check_batch(out, 2 * w, "out", rows=M, like=a)
    with _on(a):
        check("flb_mp_mul", LIB.flb_mp_mul(_ptr(a), _ptr(b), _ptr(out), w, M, _stream(stream)))
    return out


def mp_divmod(a: torch.Tensor, b: torch.Tensor, stream=None) -> Tuple[torch.Tensor, torch.Tensor]:
    """Table I div and mod (L243): (floor(a / b), a mod b); b = 0 gives (2^(32 words) - 1, a)."""
    M, w = _mp_operands(a, b)
    q, r = torch.empty_like(a), torch.empty_like(a)
    with _on(a):
        check("flb_mp_divmod", LIB.flb_mp_divmod(_ptr(a), _ptr(b), _ptr(q), _ptr(r), w, M, _stream(stream)))
    return q, r


def mp_mod(x: torch.Tensor, n: torch.Tensor, out=None, stream=None) -> torch.Tensor:
    """Table I mod(x, n): x mod n per row."""
    M, w = _mp_operands(x, n, "x", "n")
    out = torch.empty_like(x) if out is None else out
    _check_batch(out, w, "out", rows=M, like=x)
    with _on(x):
        check("flb_mp_mod", LIB.flb_mp_mod(_ptr(x), _ptr(n), _ptr(out), w, M, _stream(stream)))
    return out


def mp_mod_inv(x: torch.Tensor, n: torch.Tensor, out=None, ok=None, stream=None) -> torch.Tensor:
    """Table I mod_inv(x, n): x^-1 mod n per row (any n >= 2); 0 where no inverse exists
    (``ok`` = 0 there)."""
    M, w = _mp_operands(x, n, "x", "n")
    out = torch.empty_like(x) if out is None else out
    _check_batch(out, w, "out", rows=M, like=x)
    with _on(x):
        check("flb_mp_mod_inv", LIB.flb_mp_mod_inv(_ptr(x), _ptr(n), _ptr(out), _ptr(_mp_flag(ok, M, x)), w, M,
                                                   _stream(stream)))
    return out


# ----------------------------------------------------------------------------- host-buffer pipeline
def _np_ptr(a):
    import numpy as np
    if not isinstance(a, np.ndarray) or not a.flags["C_CONTIGUOUS"]:
        raise ValueError("host buffers must be C-contiguous numpy arrays")
    return a.ctypes.data


def pack_encrypt_host(pub: PublicKey, codec: Codec, x, seed: int = 0, ctr0: int = 0,
                      priv: Optional[PrivateKey] = None, out=None):
    """Host float32 values -> host ciphertext limbs [M, ct_words] (uint32), pipelined (PAPER Fig. 4 ①–④).
    With ``priv`` the key-holder CRT encryption is used (same bits)."""
    import numpy as np
    x = np.ascontiguousarray(x, dtype=np.float32)
    M = codec.num_plaintexts(x.shape[0])
    if out is None:
        out = np.empty((M, pub.ct_words), dtype=np.uint32)
    _check_host_out(out, (M, pub.ct_words), np.uint32, "out")
    cs = codec.struct()
    check("flb_pack_encrypt_host", LIB.flb_pack_encrypt_host(pub.handle, priv.handle if priv else None,
                                                             ctypes.byref(cs), _np_ptr(x), x.shape[0],
                                                             seed & 0xFFFFFFFFFFFFFFFF, ctr0, _np_ptr(out)))
    return out


def _check_host_out(out, shape, dtype, what):
    """A caller-supplied host output: C-contiguous numpy array of exactly this shape and dtype (it may live
    in page-locked memory, e.g. a pin_memory tensor's .numpy(): the pipeline then copies into it directly)."""
    import numpy as np
    if not isinstance(out, np.ndarray) or out.dtype != dtype or tuple(out.shape) != tuple(shape) \
            or not out.flags["C_CONTIGUOUS"]:
        raise ValueError("%s must be a C-contiguous %s array of shape %s" % (what, np.dtype(dtype).name, tuple(shape)))


def pack_encrypt_host_multi(pub: PublicKey, codec: Codec, xs, seed: int = 0, ctr0: int = 0,
                            priv: Optional[PrivateKey] = None, out=None):
    """Several host float32 arrays (e.g. one per client), each packed with its own slot alignment,
    encrypted as one pipelined batch -> host ciphertexts [sum_a ceil(len_a/S), ct_words]."""
    import numpy as np
    xs = [np.ascontiguousarray(x, dtype=np.float32) for x in xs]
    M = sum(codec.num_plaintexts(x.shape[0]) for x in xs)
    if out is None:
        out = np.empty((M, pub.ct_words), dtype=np.uint32)
    _check_host_out(out, (M, pub.ct_words), np.uint32, "out")
    ptrs = (ctypes.c_void_p * len(xs))(*[x.ctypes.data for x in xs])
    lens = (ctypes.c_size_t * len(xs))(*[x.shape[0] for x in xs])
    cs = codec.struct()
    check("flb_pack_encrypt_host_multi", LIB.flb_pack_encrypt_host_multi(pub.handle, priv.handle if priv else None,
                                                                         ctypes.byref(cs), ptrs, lens, len(xs),
                                                                         seed & 0xFFFFFFFFFFFFFFFF, ctr0,
                                                                         _np_ptr(out)))
    return out


def decrypt_unpack_host(priv: PrivateKey, codec: Codec, c, n_values: int, summands=1, out=None):
    """Host ciphertexts -> host float32 values, pipelined (PAPER Fig. 4 ⑤–⑨)."""
    import numpy as np
    c = np.ascontiguousarray(c, dtype=np.uint32)
    if c.ndim != 2 or c.shape[1] != priv.pub.ct_words or c.shape[0] < codec.num_plaintexts(n_values):
        raise ValueError("c must be [>= %d, %d] ciphertext limbs" % (codec.num_plaintexts(n_values), priv.pub.ct_words))
    if out is None:
        out = np.empty((n_values,), dtype=np.float32)
    _check_host_out(out, (n_values,), np.float32, "out")
    cs = codec.struct()
    if isinstance(summands, int):
        sp, ss = None, summands
    else:
        summands = np.ascontiguousarray(summands, dtype=np.uint32)
        sp, ss = _np_ptr(summands), 0
    check("flb_decrypt_unpack_host", LIB.flb_decrypt_unpack_host(priv.handle, priv.pub.handle, ctypes.byref(cs),
                                                                 _np_ptr(c), n_values, sp, ss, _np_ptr(out)))
    return out


def reduce_segments_host(pub: PublicKey, c, offsets, idx=None, max_segment_len: int = 0, out=None):
    """Segmented ciphertext product over host buffers."""
    import numpy as np
    c = np.ascontiguousarray(c, dtype=np.uint32)
    offsets = np.ascontiguousarray(offsets, dtype=np.int64)
    S = offsets.shape[0] - 1
    ip = None
    if idx is not None:
        idx = np.ascontiguousarray(idx, dtype=np.int64)
        ip = _np_ptr(idx)
    if c.ndim != 2 or c.shape[1] != pub.ct_words:
        raise ValueError("c must be [count, %d] ciphertext limbs" % pub.ct_words)
    if out is None:
        out = np.empty((S, pub.ct_words), dtype=np.uint32)
    _check_host_out(out, (S, pub.ct_words), np.uint32, "out")
    check("flb_reduce_segments_host", LIB.flb_reduce_segments_host(pub.handle, _np_ptr(c), c.shape[0], ip,
                                                                   _np_ptr(offsets), S, max_segment_len,
                                                                   _np_ptr(out)))
    return out


OPS = {"encrypt": 0, "decrypt": 1, "add": 2, "reduce_input": 3, "encrypt_crt": 4, "encrypt_crt_tc": 5,
       "decrypt_tc": 6, "encrypt_crt_tc_macs": 7, "decrypt_tc_macs": 8, "encrypt_tc": 9, "encrypt_tc_macs": 10}


def op_cost(key, op: str) -> Tuple[int, int]:
    """(Montgomery multiplications, CIOS limb products) per element of ``op`` (roofline accounting)."""
    mm, lp = ctypes.c_uint64(), ctypes.c_uint64()
    pub = key.handle if isinstance(key, PublicKey) else None
    priv = key.handle if isinstance(key, PrivateKey) else None
    check("flb_op_cost", LIB.flb_op_cost(pub, priv, OPS[op], ctypes.byref(mm), ctypes.byref(lp)))
    return mm.value, lp.value


def debug_tc_product(a: torch.Tensor, b: torch.Tensor, square: bool = False, stream=None) -> torch.Tensor:
    """The tensor-core Montgomery kernel's product phase alone: a_i b_i (or a_i^2) as 2w-limb rows,
    w = a.shape[1] in {32, 64, 96, 128}, at most 128 rows (debugging and parity tests).  square: 0/False =
    general product, 1/True = block squaring (one triangular diagonal square per lane), 2 = block
    squaring with the half-split diagonal square."""
    M = _check_batch(a, a.shape[1], "a")
    _check_batch(b, a.shape[1], "b", rows=M, like=a)
    out = torch.empty((M, 2 * a.shape[1]), dtype=torch.int32, device=a.device)
    with _on(a):
        check("flb_debug_tc_product", LIB.flb_debug_tc_product(_ptr(a), _ptr(b), _ptr(out), M, a.shape[1],
                                                               int(square), _stream(stream)))
    return out


def debug_mont_mul(pub: PublicKey, a: torch.Tensor, b: torch.Tensor, out: Optional[torch.Tensor] = None,
                   stream=None) -> torch.Tensor:
    """a b R^-1 mod n^2 (the Montgomery primitive of PAPER Alg. 2)."""
    M = _check_batch(a, pub.ct_words, "a")
    _check_batch(b, pub.ct_words, "b", rows=M, like=a)
    if out is None:
        out = torch.empty_like(a)
    _check_batch(out, pub.ct_words, "out", rows=M, like=a)
    with _on(a):
        check("flb_debug_mont_mul", LIB.flb_debug_mont_mul(pub.handle, _ptr(a), _ptr(b), _ptr(out), M,
                                                           _stream(stream)))
    return out
