"""B200-native SNP comparison (Binder, Low & Popovici, IPDPS-W 2019) — Python binding.

A thin layer over the C ABI of ``libsnp.so`` (``include/snp.h``): it checks
tensor devices/dtypes, allocates outputs and workspace with torch (the library
itself allocates nothing), passes raw pointers plus the current CUDA stream,
and raises :class:`SnpError` on a non-zero status.  Every step of the path runs
in the library's CUDA kernels; there is no CPU or PyTorch fallback.

Dtypes: packed bit matrices are ``torch.uint64`` ``[rows][ld]`` (ld even, see
:func:`snp_words`); counts are ``torch.uint32``; r2 / D' are ``torch.float32``.
"""
from __future__ import annotations

import ctypes

import torch

from ._lib import SnpError, check, lib, status_string  # noqa: F401

__all__ = [
    "SnpError", "OPS", "VARIANTS", "snp_words", "snp_ld_workspace_bytes",
    "snp_fastid_workspace_bytes", "snp_pack", "snp_pack_popc", "snp_row_popc", "snp_ld_counts",
    "snp_ld_r2", "snp_fastid", "snp_fastid_best", "snp_fastid_search",
    "snp_fastid_search_workspace_bytes", "snp_fastid_threshold", "snp_fastid_threshold_workspace_bytes",
    "snp_shard_plan", "snp_shard_plan_sym", "snp_sym_tiles",
    "snp_ld_sym_workspace_bytes", "snp_ld_sym", "snp_sym_unpack", "snp_set_variant",
    "snp_last_variant", "snp_last_kernel", "snp_launch_count", "status_string",
]

OPS = {"and": 0, "xor": 1, "andnot": 2, "notand": 3}
VARIANTS = {"auto": 0, "popc": 1, "tc": 2}


def _op(op) -> int:
    if isinstance(op, str):
        if op not in OPS:
            raise SnpError(4, "op", op)
        return OPS[op]
    return int(op)


def _stream(stream) -> ctypes.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t) -> ctypes.c_void_p:
    return ctypes.c_void_p(0 if t is None else t.data_ptr())


def _dev_tensor(t, name, dtypes):
    if t is None:
        return
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype not in dtypes:
        raise TypeError(f"{name} must have dtype in {dtypes}, got {t.dtype}")
    if t.dim() >= 1 and t.stride(-1) != 1:
        raise ValueError(f"{name} must be contiguous along its last dimension")


def _ld(t) -> int:
    return t.stride(0) if t.dim() == 2 else t.shape[-1]


_WORD_DTYPES = (torch.uint64, torch.int64)
_U32 = (torch.uint32, torch.int32)


def snp_words(nbits: int) -> int:
    """Recommended packed leading dimension (uint64 words) for nbits."""
    return int(lib().snp_words(int(nbits)))


def snp_ld_workspace_bytes(m: int, n: int, nbits: int) -> int:
    return int(lib().snp_ld_workspace_bytes(int(m), int(n), int(nbits)))


def snp_fastid_workspace_bytes(nq: int, nd: int, nbits: int, op="xor") -> int:
    return int(lib().snp_fastid_workspace_bytes(int(nq), int(nd), int(nbits), _op(op)))


def _workspace(nbytes: int, device) -> torch.Tensor | None:
    if nbytes == 0:
        return None
    return torch.empty(nbytes, dtype=torch.uint8, device=device)


def snp_pack(g: torch.Tensor, nbits: int | None = None, ldw: int | None = None,
             out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a1: uint8 genotypes [rows][>= nbits] (non-zero = minor allele) -> packed uint64."""
    _dev_tensor(g, "g", (torch.uint8, torch.bool))
    rows = g.shape[0]
    nbits = g.shape[1] if nbits is None else int(nbits)
    if out is None:
        ldw = snp_words(nbits) if ldw is None else int(ldw)
        out = torch.empty((rows, ldw), dtype=torch.uint64, device=g.device)
    _dev_tensor(out, "out", _WORD_DTYPES)
    check(lib().snp_pack(_ptr(g), rows, nbits, _ld(g), _ptr(out), _ld(out), _stream(stream)), "snp_pack")
    return out


def snp_pack_popc(g: torch.Tensor, nbits: int | None = None, ldw: int | None = None,
                  out: torch.Tensor | None = None, popc: torch.Tensor | None = None,
                  stream=None) -> tuple[torch.Tensor, torch.Tensor]:
    """a1 + a2 fused: packed uint64 rows and their uint32 popcounts from one pass over g."""
    _dev_tensor(g, "g", (torch.uint8, torch.bool))
    rows = g.shape[0]
    nbits = g.shape[1] if nbits is None else int(nbits)
    if out is None:
        ldw = snp_words(nbits) if ldw is None else int(ldw)
        out = torch.empty((rows, ldw), dtype=torch.uint64, device=g.device)
    if popc is None:
        popc = torch.empty(rows, dtype=torch.uint32, device=g.device)
    _dev_tensor(out, "out", _WORD_DTYPES)
    _dev_tensor(popc, "popc", _U32)
    check(lib().snp_pack_popc(_ptr(g), rows, nbits, _ld(g), _ptr(out), _ld(out), _ptr(popc), _stream(stream)),
          "snp_pack_popc")
    return out, popc


def snp_row_popc(x: torch.Tensor, nbits: int, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a2: per-row popcount of the first nbits bits."""
    _dev_tensor(x, "x", _WORD_DTYPES)
    if out is None:
        out = torch.empty(x.shape[0], dtype=torch.uint32, device=x.device)
    _dev_tensor(out, "out", _U32)
    check(lib().snp_row_popc(_ptr(x), x.shape[0], int(nbits), _ld(x), _ptr(out), _stream(stream)),
          "snp_row_popc")
    return out


def snp_ld_counts(A: torch.Tensor, B: torch.Tensor, nbits: int, C: torch.Tensor | None = None,
                  accumulate: bool = False, ws: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a3: C[i][j] (+)= popc(A_i & B_j) over nbits (Eq. 1)."""
    _dev_tensor(A, "A", _WORD_DTYPES)
    _dev_tensor(B, "B", _WORD_DTYPES)
    m, n = A.shape[0], B.shape[0]
    if C is None:
        C = (torch.zeros if accumulate else torch.empty)((m, n), dtype=torch.uint32, device=A.device)
    _dev_tensor(C, "C", _U32)
    need = snp_ld_workspace_bytes(m, n, nbits)
    if ws is None:
        ws = _workspace(need, A.device)
    check(lib().snp_ld_counts(_ptr(A), m, _ld(A), _ptr(B), n, _ld(B), int(nbits), _ptr(C), _ld(C),
                              1 if accumulate else 0, _ptr(ws), 0 if ws is None else ws.numel(),
                              _stream(stream)), "snp_ld_counts")
    return C


def snp_ld_r2(A: torch.Tensor, B: torch.Tensor, nbits: int, popA=None, popB=None,
              r2: torch.Tensor | None = None, dprime: torch.Tensor | bool | None = None,
              counts: torch.Tensor | bool | None = None, ws: torch.Tensor | None = None,
              stream=None):
    """a3+a5: r2 (and optionally D', nAB counts) for every SNP pair.

    Returns (r2, dprime_or_None, counts_or_None).  Pass dprime=True / counts=True
    to have them allocated."""
    _dev_tensor(A, "A", _WORD_DTYPES)
    _dev_tensor(B, "B", _WORD_DTYPES)
    m, n = A.shape[0], B.shape[0]
    dev = A.device
    if r2 is None:
        r2 = torch.empty((m, n), dtype=torch.float32, device=dev)
    if dprime is True:
        dprime = torch.empty((m, n), dtype=torch.float32, device=dev)
    elif dprime is False:
        dprime = None
    if counts is True:
        counts = torch.empty((m, n), dtype=torch.uint32, device=dev)
    elif counts is False:
        counts = None
    _dev_tensor(r2, "r2", (torch.float32,))
    _dev_tensor(dprime, "dprime", (torch.float32,))
    _dev_tensor(counts, "counts", _U32)
    _dev_tensor(popA, "popA", _U32)
    _dev_tensor(popB, "popB", _U32)
    need = snp_ld_workspace_bytes(m, n, nbits)
    if ws is None:
        ws = _workspace(need, dev)
    check(lib().snp_ld_r2(_ptr(A), m, _ld(A), _ptr(popA), _ptr(B), n, _ld(B), _ptr(popB), int(nbits),
                          _ptr(r2), _ptr(dprime), _ptr(counts), _ld(r2), _ptr(ws),
                          0 if ws is None else ws.numel(), _stream(stream)), "snp_ld_r2")
    return r2, dprime, counts


def snp_fastid(Q: torch.Tensor, D: torch.Tensor, nbits: int, op="xor", out: torch.Tensor | None = None,
               popQ=None, popD=None, accumulate: bool = False, ws: torch.Tensor | None = None,
               stream=None) -> torch.Tensor:
    """a3+a4: out[i][j] (+)= popc(Q_i op D_j), op in and|xor|andnot|notand (Eqs. 1-3)."""
    _dev_tensor(Q, "Q", _WORD_DTYPES)
    _dev_tensor(D, "D", _WORD_DTYPES)
    opi = _op(op)
    nq, nd = Q.shape[0], D.shape[0]
    if out is None:
        out = (torch.zeros if accumulate else torch.empty)((nq, nd), dtype=torch.uint32, device=Q.device)
    _dev_tensor(out, "out", _U32)
    _dev_tensor(popQ, "popQ", _U32)
    _dev_tensor(popD, "popD", _U32)
    need = lib().snp_fastid_workspace_bytes(nq, nd, int(nbits), opi)
    if ws is None:
        ws = _workspace(int(need), Q.device)
    check(lib().snp_fastid(_ptr(Q), nq, _ld(Q), _ptr(popQ), _ptr(D), nd, _ld(D), _ptr(popD), int(nbits),
                           opi, _ptr(out), _ld(out), 1 if accumulate else 0, _ptr(ws),
                           0 if ws is None else ws.numel(), _stream(stream)), "snp_fastid")
    return out


def snp_fastid_best(counts: torch.Tensor, index_base: int = 0, nd: int | None = None,
                    best_count: torch.Tensor | None = None, best_index: torch.Tensor | None = None,
                    stream=None):
    """a6: per query (min count, lowest index attaining it + index_base)."""
    _dev_tensor(counts, "counts", _U32)
    nq = counts.shape[0]
    nd = counts.shape[1] if nd is None else int(nd)
    if best_count is None:
        best_count = torch.empty(nq, dtype=torch.uint32, device=counts.device)
    if best_index is None:
        best_index = torch.empty(nq, dtype=torch.int64, device=counts.device)
    check(lib().snp_fastid_best(_ptr(counts), nq, nd, _ld(counts), int(index_base), _ptr(best_count),
                                _ptr(best_index), _stream(stream)), "snp_fastid_best")
    return best_count, best_index


def snp_fastid_search_workspace_bytes(nq: int, nd: int, nbits: int, nops: int) -> int:
    """Bytes of the search workspace; allocate it zero-filled (torch.zeros): the library
    keeps it zero-filled from call to call."""
    return int(lib().snp_fastid_search_workspace_bytes(int(nq), int(nd), int(nbits), int(nops)))


def snp_fastid_search(Q: torch.Tensor, D: torch.Tensor, nbits: int, ops=("xor", "andnot"),
                      counts=True, best=True, index_base: int = 0, ldo: int | None = None,
                      ws: torch.Tensor | None = None, popD: torch.Tensor | None = None, stream=None):
    """f1: one pass over D for every op in ops -> (counts list, best list).

    counts: True (allocate [nq][nd] uint32 per op), False (none) or a list of
    tensors/None per op.  best: True/False or a list of (best_count, best_index)
    pairs / None per op.  Returns (counts_list, best_list), entries None where not
    requested."""
    _dev_tensor(Q, "Q", _WORD_DTYPES)
    _dev_tensor(D, "D", _WORD_DTYPES)
    if isinstance(ops, (str, int)):
        ops = (ops,)
    opi = [_op(o) for o in ops]
    k = len(opi)
    nq, nd = Q.shape[0], D.shape[0]
    dev = Q.device
    if counts is True:
        counts = [torch.empty((nq, nd if ldo is None else ldo), dtype=torch.uint32, device=dev) for _ in opi]
    elif counts is False or counts is None:
        counts = [None] * k
    if best is True:
        best = [(torch.empty(nq, dtype=torch.uint32, device=dev), torch.empty(nq, dtype=torch.int64, device=dev))
                for _ in opi]
    elif best is False or best is None:
        best = [None] * k
    if len(counts) != k or len(best) != k:
        raise ValueError("counts / best must have one entry per op")
    for c in counts:
        _dev_tensor(c, "counts", _U32)
    for b in best:
        if b is not None:
            _dev_tensor(b[0], "best_count", _U32)
            _dev_tensor(b[1], "best_index", (torch.int64,))
    ld = next((_ld(c) for c in counts if c is not None), nd if ldo is None else int(ldo))
    P = ctypes.c_void_p * k
    ops_arr = (ctypes.c_int * k)(*opi)
    c_arr = P(*[_ptr(c) for c in counts])
    bc_arr = P(*[_ptr(None if b is None else b[0]) for b in best])
    bi_arr = P(*[_ptr(None if b is None else b[1]) for b in best])
    need = snp_fastid_search_workspace_bytes(nq, nd, nbits, k)
    if ws is None:   # zero-filled on first use (snp.h); every call leaves it zero-filled
        ws = None if need == 0 else torch.zeros(need, dtype=torch.uint8, device=dev)
    any_best = any(b is not None for b in best)
    _dev_tensor(popD, "popD", _U32)
    if popD is not None and popD.numel() < nd:
        raise ValueError("popD needs one popcount per database row")
    check(lib().snp_fastid_search(_ptr(Q), nq, _ld(Q), _ptr(D), nd, _ld(D), _ptr(popD), int(nbits), k,
                                  ctypes.cast(ops_arr, ctypes.c_void_p), ctypes.cast(c_arr, ctypes.c_void_p), ld,
                                  ctypes.cast(bc_arr, ctypes.c_void_p) if any_best else None,
                                  ctypes.cast(bi_arr, ctypes.c_void_p) if any_best else None,
                                  int(index_base), _ptr(ws), 0 if ws is None else ws.numel(), _stream(stream)),
          "snp_fastid_search")
    return counts, best


def snp_fastid_threshold_workspace_bytes(nq: int, nd: int, nbits: int, op="xor") -> int:
    return int(lib().snp_fastid_threshold_workspace_bytes(int(nq), int(nd), int(nbits), _op(op)))


def snp_fastid_threshold(Q: torch.Tensor, D: torch.Tensor, nbits: int, op="xor", tau: int = 0,
                         capacity: int = 1 << 16, index_base: int = 0, popD=None, ws=None, stream=None):
    """f1 threshold form: every (query, database row) with count <= tau.

    Returns (query, count, index, total): int64 / uint32-in-int64 / int64 device tensors of the
    stored matches (at most `capacity`, unspecified order) and the total number of matches
    (host int; > capacity means the list was truncated)."""
    _dev_tensor(Q, "Q", _WORD_DTYPES)
    _dev_tensor(D, "D", _WORD_DTYPES)
    _dev_tensor(popD, "popD", _U32)
    opi = _op(op)
    nq, nd = Q.shape[0], D.shape[0]
    dev = Q.device
    m = torch.empty((max(1, int(capacity)), 2), dtype=torch.int64, device=dev)   # 16-byte snp_match
    total = torch.zeros(1, dtype=torch.int64, device=dev)
    if ws is None:
        ws = _workspace(snp_fastid_threshold_workspace_bytes(nq, nd, nbits, opi), dev)
    check(lib().snp_fastid_threshold(_ptr(Q), nq, _ld(Q), _ptr(D), nd, _ld(D), _ptr(popD), int(nbits), opi,
                                     int(tau), int(index_base), _ptr(m), int(capacity), _ptr(total), _ptr(ws),
                                     0 if ws is None else ws.numel(), _stream(stream)), "snp_fastid_threshold")
    n = int(total.item())
    k = min(n, int(capacity))
    w0 = m[:k, 0]
    return w0 & 0xFFFFFFFF, (w0 >> 32) & 0xFFFFFFFF, m[:k, 1], n


def snp_shard_plan(rows: int, world: int, align: int = 128) -> list[int]:
    """e: contiguous, align-multiple row ranges per rank (host only)."""
    arr = (ctypes.c_int64 * (int(world) + 1))() if world >= 1 else (ctypes.c_int64 * 1)()
    check(lib().snp_shard_plan(int(rows), int(world), int(align), ctypes.cast(arr, ctypes.c_void_p)),
          "snp_shard_plan")
    return [int(v) for v in arr]


SYM_TILE = 128


def snp_sym_tiles(m: int) -> int:
    """f3: number of 128 x 128 tiles in the upper triangle of an m x m self-LD output."""
    return int(lib().snp_sym_tiles(int(m)))


def snp_shard_plan_sym(m: int, world: int) -> list[int]:
    """e + f3: triangle-balanced contiguous tile ranges per rank (host only)."""
    arr = (ctypes.c_int64 * (max(1, int(world)) + 1))()
    check(lib().snp_shard_plan_sym(int(m), int(world), ctypes.cast(arr, ctypes.c_void_p)), "snp_shard_plan_sym")
    return [int(v) for v in arr][:int(world) + 1]


def snp_ld_sym_workspace_bytes(m: int, nbits: int) -> int:
    return int(lib().snp_ld_sym_workspace_bytes(int(m), int(nbits)))


def snp_ld_sym(A: torch.Tensor, nbits: int, tile_lo: int = 0, tile_hi: int | None = None, popA=None,
               r2: torch.Tensor | bool | None = True, dprime: torch.Tensor | bool | None = None,
               counts: torch.Tensor | bool | None = None, ws: torch.Tensor | None = None, stream=None):
    """f3: self-LD tiles [tile_lo, tile_hi) of the row-major upper triangle, each a dense
    128 x 128 block ([tiles][128][128] outputs).  Returns (r2, dprime, counts), None where
    not requested (True allocates)."""
    _dev_tensor(A, "A", _WORD_DTYPES)
    m = A.shape[0]
    tile_hi = snp_sym_tiles(m) if tile_hi is None else int(tile_hi)
    nt = max(0, tile_hi - int(tile_lo))
    dev = A.device

    def _out(x, dt):
        if x is True:
            return torch.empty((nt, SYM_TILE, SYM_TILE), dtype=dt, device=dev)
        return None if x is False else x
    r2, dprime, counts = _out(r2, torch.float32), _out(dprime, torch.float32), _out(counts, torch.uint32)
    _dev_tensor(r2, "r2", (torch.float32,))
    _dev_tensor(dprime, "dprime", (torch.float32,))
    _dev_tensor(counts, "counts", _U32)
    _dev_tensor(popA, "popA", _U32)
    for t in (r2, dprime, counts):
        if t is not None and t.numel() < nt * SYM_TILE * SYM_TILE:
            raise ValueError("snp_ld_sym outputs need (tile_hi - tile_lo) * 128 * 128 elements")
    if ws is None:
        ws = _workspace(snp_ld_sym_workspace_bytes(m, nbits), dev)
    check(lib().snp_ld_sym(_ptr(A), m, _ld(A), _ptr(popA), int(nbits), int(tile_lo), tile_hi, _ptr(r2), _ptr(dprime),
                           _ptr(counts), _ptr(ws), 0 if ws is None else ws.numel(), _stream(stream)), "snp_ld_sym")
    return r2, dprime, counts


def snp_sym_unpack(tiles: torch.Tensor, m: int, tile_lo: int = 0, tile_hi: int | None = None,
                   out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """f3: packed-triangle tiles (any 4-byte dtype) -> the full symmetric m x m matrix."""
    if not tiles.is_cuda or tiles.element_size() != 4:
        raise TypeError("tiles must be a CUDA tensor of 4-byte elements")
    tile_hi = snp_sym_tiles(m) if tile_hi is None else int(tile_hi)
    if out is None:
        out = torch.empty((m, m), dtype=tiles.dtype, device=tiles.device)
    if out.element_size() != 4 or out.stride(-1) != 1:
        raise TypeError("out must have 4-byte elements, contiguous rows")
    check(lib().snp_sym_unpack(_ptr(tiles), int(m), int(tile_lo), tile_hi, _ptr(out), _ld(out), _stream(stream)),
          "snp_sym_unpack")
    return out


def snp_set_variant(variant) -> None:
    v = VARIANTS[variant] if isinstance(variant, str) else int(variant)
    check(lib().snp_set_variant(v), "snp_set_variant")


def snp_launch_count() -> int:
    """Cumulative number of kernels libsnp.so launched in this process."""
    return int(lib().snp_launch_count())


KERNELS = {0: "none", 1: "popc", 2: "tc_i8", 3: "tc_mxf4", 4: "fastid_mxf4", 5: "tc_mxf4_sym", 6: "popc_stream",
           7: "tc_mxf4_sym_pair", 8: "tc_mxf4_pair"}


def snp_last_kernel() -> str:
    """Kernel family of the most recent compute call on this thread."""
    return KERNELS.get(int(lib().snp_last_kernel()), "?")


def snp_last_variant() -> str:
    v = int(lib().snp_last_variant())
    return {0: "none", 1: "popc", 2: "tc"}.get(v, str(v))
