"""CPU oracle for the SNP-comparison hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_ipps_binderlp19_b200``) never imports it, and it imports nothing
from the product.

The arithmetic lives in ``snp_oracle.c`` (plain bit-by-bit loops on unpacked
0/1 bytes, see its header for the paper readings R1-R4 and citations).  This
module only marshals numpy arrays into it.  If the shared object is missing it
is compiled here with gcc (``__graft_entry__.build()`` also compiles it).

Parity status of each function (DESIGN.md §3 lists the pins):
  unpack / pack      pinned (hand examples App. C, round trip, padding zero)
  row_popc           pinned (numpy sum, closed form popcount(i))
  counts AND/XOR/    pinned (numpy int matmul, scipy hamming, exhaustive closed
    ANDNOT/NOTAND      forms popcount(i&j) ..., identities, hand examples)
  ld (r2, D')        pinned (np.corrcoef^2, textbook D' cases, hand examples)
  best               pinned (brute-force argmin on tiny inputs, planted matches)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "snp_oracle.c")
_LIB = os.path.join(_HERE, "libsnp_oracle.so")
_lock = threading.Lock()
_lib = None

OPS = {"and": 0, "xor": 1, "andnot": 2, "notand": 3}


def build(force: bool = False) -> str:
    """Compile snp_oracle.c into libsnp_oracle.so (gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i64, p = ctypes.c_int64, ctypes.c_void_p
            lib.oracle_unpack.argtypes = [p, i64, i64, i64, p, i64]
            lib.oracle_pack.argtypes = [p, i64, i64, i64, p, i64]
            lib.oracle_row_popc.argtypes = [p, i64, i64, i64, p]
            lib.oracle_counts.argtypes = [p, i64, i64, p, i64, i64, i64, ctypes.c_int, p, i64]
            lib.oracle_counts.restype = ctypes.c_int
            lib.oracle_ld.argtypes = [p, i64, i64, p, i64, i64, i64, p, p, p, i64]
            lib.oracle_ld.restype = ctypes.c_int
            lib.oracle_ld_from_counts.argtypes = [i64, i64, i64, i64, p, p]
            lib.oracle_best.argtypes = [p, i64, i64, i64, i64, p, p]
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _g(a) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.uint8)
    if a.ndim != 2:
        raise ValueError("genotype matrix must be 2-D [rows][nbits]")
    return a


def unpack(packed: np.ndarray, nbits: int) -> np.ndarray:
    """Packed uint64 [rows][ldw] -> uint8 0/1 [rows][nbits] (reading R1)."""
    packed = np.ascontiguousarray(packed, dtype=np.uint64)
    rows, ldw = packed.shape
    g = np.empty((rows, nbits), dtype=np.uint8)
    if rows and nbits:
        _load().oracle_unpack(_ptr(packed), rows, nbits, ldw, _ptr(g), nbits)
    return g


def pack(g, ldw: int | None = None) -> np.ndarray:
    """uint8 [rows][nbits] (non-zero = minor) -> uint64 [rows][ldw], zero padded."""
    g = _g(g)
    rows, nbits = g.shape
    if ldw is None:
        ldw = (nbits + 63) // 64
    out = np.empty((rows, ldw), dtype=np.uint64)
    if rows:
        _load().oracle_pack(_ptr(g), rows, nbits, nbits, _ptr(out), ldw)
    return out


def row_popc(g) -> np.ndarray:
    g = _g(g)
    rows, nbits = g.shape
    out = np.empty(rows, dtype=np.uint32)
    if rows:
        _load().oracle_row_popc(_ptr(g), rows, nbits, nbits, _ptr(out))
    return out


def counts(ga, gb, op: str = "and") -> np.ndarray:
    """C[i][j] = sum_k op(ga[i,k], gb[j,k]) bit by bit (Eqs. 1-3)."""
    ga, gb = _g(ga), _g(gb)
    if ga.shape[1] != gb.shape[1]:
        raise ValueError("nbits mismatch")
    m, nbits = ga.shape
    n = gb.shape[0]
    c = np.zeros((m, n), dtype=np.uint32)
    if m and n:
        rc = _load().oracle_counts(_ptr(ga), m, nbits, _ptr(gb), n, nbits, nbits, OPS[op], _ptr(c), n)
        if rc != 0:
            raise ValueError(op)
    return c


def ld(ga, gb):
    """(r2 float64, dprime float64, nAB uint32) for every pair (reading R3)."""
    ga, gb = _g(ga), _g(gb)
    if ga.shape[1] != gb.shape[1]:
        raise ValueError("nbits mismatch")
    m, nbits = ga.shape
    n = gb.shape[0]
    r2 = np.zeros((m, n), dtype=np.float64)
    dp = np.zeros((m, n), dtype=np.float64)
    nab = np.zeros((m, n), dtype=np.uint32)
    if m and n:
        rc = _load().oracle_ld(_ptr(ga), m, nbits, _ptr(gb), n, nbits, nbits, _ptr(r2), _ptr(dp), _ptr(nab), n)
        if rc != 0:
            raise ValueError("nbits must be >= 1")
    return r2, dp, nab


def ld_from_counts(n: int, na: int, nb: int, nab: int):
    r2 = ctypes.c_double()
    dp = ctypes.c_double()
    _load().oracle_ld_from_counts(n, na, nb, nab, ctypes.byref(r2), ctypes.byref(dp))
    return r2.value, dp.value


def best(c, index_base: int = 0):
    """Per query row: (min count uint32, lowest index attaining it + index_base)."""
    c = np.ascontiguousarray(c, dtype=np.uint32)
    nq, nd = c.shape
    b = np.empty(nq, dtype=np.uint32)
    idx = np.empty(nq, dtype=np.int64)
    if nq:
        _load().oracle_best(_ptr(c), nq, nd, nd, index_base, _ptr(b), _ptr(idx))
    return b, idx
