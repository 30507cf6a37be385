"""Boundary tests that need no GPU: the C-ABI library loads, exports every symbol
include/snp.h declares, and validates arguments synchronously (before touching
CUDA).  Host-only logic (snp_words, snp_shard_plan) is checked here too."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "snp.h")

OK, E_NULL, E_SHAPE, E_ALIGN, E_OP, E_RANGE, E_WORKSPACE, E_ARCH, E_CUDA = range(9)


def declared_symbols():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(snp_[a-z0-9_]+)\s*\(", text)))


def test_header_declares_expected_calls():
    syms = declared_symbols()
    for name in ("snp_pack", "snp_pack_popc", "snp_row_popc", "snp_ld_counts", "snp_ld_r2", "snp_fastid",
                 "snp_fastid_best", "snp_shard_plan", "snp_words", "snp_status_string"):
        assert name in syms


def test_library_exports_every_declared_symbol(snplib):
    L = snplib.lib()
    from paper_conf_ipps_binderlp19_b200._lib import SIGNATURES
    for name in declared_symbols():
        assert hasattr(L, name), name
        assert name in SIGNATURES, f"binding lacks {name}"
    # and the binding exposes a Python function of the same name for each call
    for name in declared_symbols():
        if name in ("snp_status_string", "snp_last_cuda_error"):
            continue
        assert hasattr(snplib, name), name


def test_library_is_sm100a_only(snplib):
    import subprocess
    from paper_conf_ipps_binderlp19_b200._lib import LIB_PATH
    out = subprocess.run(["cuobjdump", "--list-elf", LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "sm_90" not in out and "sm_80" not in out


def test_snp_words():
    from paper_conf_ipps_binderlp19_b200 import snp_words
    assert snp_words(0) == 0 and snp_words(-5) == 0
    assert snp_words(1) == 8 and snp_words(512) == 8 and snp_words(513) == 16
    assert snp_words(4096) == 64 and snp_words(16384) == 256


@pytest.mark.parametrize("rows,world,align", [(0, 1, 128), (1, 1, 128), (1000, 3, 128),
                                              (32768, 8, 128), (20_000_000, 8, 128),
                                              (129, 2, 128), (5, 8, 1), (7, 8, 2)])
def test_shard_plan_properties(snplib, rows, world, align):
    b = snplib.snp_shard_plan(rows, world, align)
    assert len(b) == world + 1 and b[0] == 0 and b[-1] == rows
    assert all(b[r] <= b[r + 1] for r in range(world))               # contiguous, disjoint
    assert all(x % align == 0 or x == rows for x in b)                # aligned (or the end)
    blocks = [(b[r + 1] - b[r] + align - 1) // align for r in range(world)]
    assert max(blocks) - min(blocks) <= 1 or rows < align * world    # balanced
    assert sum(b[r + 1] - b[r] for r in range(world)) == rows         # covers
    assert b == snplib.snp_shard_plan(rows, world, align)             # deterministic


def test_shard_plan_bad_args(snplib):
    L = snplib.lib()
    arr = (ctypes.c_int64 * 4)()
    p = ctypes.cast(arr, ctypes.c_void_p)
    assert L.snp_shard_plan(10, 0, 128, p) == E_RANGE
    assert L.snp_shard_plan(10, 2, 0, p) == E_RANGE
    assert L.snp_shard_plan(-1, 2, 128, p) == E_RANGE
    assert L.snp_shard_plan(10, 2, 128, None) == E_NULL


def test_status_strings(snplib):
    L = snplib.lib()
    for s in range(9):
        assert L.snp_status_string(s).decode().startswith("SNP_")
    assert b"unknown" in L.snp_status_string(99)


FAKE = 0x10000  # a 16-byte aligned non-NULL address: never dereferenced (validation fails first)


def test_validation_errors_before_launch(snplib):
    L = snplib.lib()
    p = ctypes.c_void_p(FAKE)
    odd = ctypes.c_void_p(FAKE + 8)
    null = None
    # snp_ld_counts(A, m, lda, B, n, ldb, nbits, C, ldc, acc, ws, ws_bytes, stream)
    assert L.snp_ld_counts(null, 4, 2, p, 4, 2, 100, p, 4, 0, null, 0, null) == E_NULL
    assert L.snp_ld_counts(p, -1, 2, p, 4, 2, 100, p, 4, 0, null, 0, null) == E_SHAPE
    assert L.snp_ld_counts(p, 4, 1, p, 4, 2, 100, p, 4, 0, null, 0, null) == E_SHAPE   # lda < words
    assert L.snp_ld_counts(p, 4, 3, p, 4, 2, 100, p, 4, 0, null, 0, null) == E_ALIGN   # odd ld
    assert L.snp_ld_counts(odd, 4, 2, p, 4, 2, 100, p, 4, 0, null, 0, null) == E_ALIGN
    assert L.snp_ld_counts(p, 4, 2, p, 4, 2, 0, p, 4, 0, null, 0, null) == E_SHAPE     # nbits < 1
    assert L.snp_ld_counts(p, 4, 2, p, 4, 2, 100, p, 3, 0, null, 0, null) == E_SHAPE   # ldc < n
    assert L.snp_ld_counts(p, 4, 2, p, 4, 2, 100, null, 4, 0, null, 0, null) == E_NULL
    assert L.snp_ld_counts(p, 4, 2, p, 4, 2, 1 << 33, p, 4, 0, null, 0, null) == E_RANGE
    # zero-sized problems are valid no-ops
    assert L.snp_ld_counts(p, 0, 2, p, 4, 2, 100, null, 4, 0, null, 0, null) == OK
    assert L.snp_fastid(p, 4, 2, null, p, 0, 2, null, 100, 1, null, 0, 0, null, 0, null) == OK
    # bad op
    assert L.snp_fastid(p, 4, 2, null, p, 4, 2, null, 100, 7, p, 4, 0, null, 0, null) == E_OP
    # r2 requires the workspace returned by the query
    assert L.snp_ld_r2(p, 4, 2, null, p, 4, 2, null, 100, p, null, null, 4, null, 0, null) == E_WORKSPACE
    # pack validation
    assert L.snp_pack(null, 3, 100, 100, p, 2, null) == E_NULL
    assert L.snp_pack(p, 3, 100, 99, p, 2, null) == E_SHAPE
    assert L.snp_pack(p, 3, 100, 100, p, 1, null) == E_SHAPE
    assert L.snp_pack(p, 3, 100, 100, odd, 2, null) == E_ALIGN
    # best
    assert L.snp_fastid_best(p, 2, 10, 5, 0, p, p, null) == E_SHAPE
    assert L.snp_set_variant(9) == E_OP


def test_valid_call_without_b200_is_refused(snplib):
    """No fallback: on a host without a compute-capability-10.0 GPU a valid call
    returns SNP_E_ARCH (this CPU box has no GPU at all)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    L = snplib.lib()
    p = ctypes.c_void_p(FAKE)
    ws = snplib.snp_ld_workspace_bytes(4, 4, 100)
    assert L.snp_ld_counts(p, 4, 2, p, 4, 2, 100, p, 4, 0, p, ws, None) == E_ARCH
    with pytest.raises(snplib.SnpError):
        snplib._lib.check(E_ARCH, "x")


def test_workspace_queries(snplib):
    assert snplib.snp_ld_workspace_bytes(0, 5, 100) == 0
    assert snplib.snp_ld_workspace_bytes(300, 500, 100) >= 4 * 800
    assert snplib.snp_fastid_workspace_bytes(0, 5, 100) == 0


def test_search_validation_before_launch(snplib):
    """snp_fastid_search (f1): argument checks happen synchronously, before CUDA."""
    L = snplib.lib()
    p = ctypes.c_void_p(FAKE)
    null = None
    P2 = ctypes.c_void_p * 2
    ops = (ctypes.c_int * 2)(1, 2)
    badops = (ctypes.c_int * 2)(1, 9)
    outs = P2(FAKE, FAKE)
    half = P2(FAKE, None)
    cast = lambda a: ctypes.cast(a, ctypes.c_void_p)   # noqa: E731
    # (Q, nq, ldq, D, nd, ldd, nbits, nops, ops, counts, ldo, best_count, best_index, base, ws, ws_bytes, stream)
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 0, cast(ops), null, 9, null, null, 0, p, 1 << 20, null) == E_OP
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 5, cast(ops), null, 9, null, null, 0, p, 1 << 20, null) == E_OP
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(badops), null, 9, null, null, 0, p, 1 << 20,
                               null) == E_OP
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, null, null, 9, null, null, 0, p, 1 << 20, null) == E_NULL
    # best_count array without best_index array, and a half-set (count, index) pair
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(ops), null, 9, cast(outs), null, 0, p, 1 << 20,
                               null) == E_NULL
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(ops), null, 9, cast(outs), cast(half), 0, p,
                               1 << 20, null) == E_NULL
    # counts need ldo >= nd; packed operands validated like snp_fastid
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(ops), cast(outs), 8, null, null, 0, p, 1 << 20,
                               null) == E_SHAPE
    assert L.snp_fastid_search(p, 4, 1, p, 9, 2, null, 100, 2, cast(ops), cast(outs), 9, null, null, 0, p, 1 << 20,
                               null) == E_SHAPE
    assert L.snp_fastid_search(p, 4, 2, p, 1 << 32, 2, null, 100, 2, cast(ops), cast(outs), 1 << 32, null, null, 0, p,
                               1 << 20, null) == E_RANGE
    # nothing requested / nq == 0: valid no-ops
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(ops), null, 9, null, null, 0, null, 0, null) == OK
    assert L.snp_fastid_search(p, 0, 2, p, 9, 2, null, 100, 2, cast(ops), cast(outs), 9, null, null, 0, null, 0,
                               null) == OK
    # the workspace is always required when there is work
    assert L.snp_fastid_search(p, 4, 2, p, 9, 2, null, 100, 2, cast(ops), cast(outs), 9, null, null, 0, null, 0,
                               null) == E_WORKSPACE
    assert snplib.snp_fastid_search_workspace_bytes(4, 9, 100, 2) >= 2 * 4 * 8
    assert snplib.snp_fastid_search_workspace_bytes(4, 0, 100, 2) >= 2 * 4 * 8
    assert snplib.snp_fastid_search_workspace_bytes(0, 9, 100, 2) == 0


@pytest.mark.parametrize("m,world", [(0, 1), (1, 1), (128, 3), (300, 2), (2048, 8), (32768, 8), (32768, 7),
                                     (100_000, 5), (129, 8)])
def test_shard_plan_sym_properties(snplib, m, world):
    """e + f3: contiguous tile ranges covering every upper-triangle tile exactly once,
    tile counts balanced within one, deterministic."""
    T = -(-m // 128)
    total = T * (T + 1) // 2
    assert snplib.snp_sym_tiles(m) == total
    b = snplib.snp_shard_plan_sym(m, world)
    assert len(b) == world + 1 and b[0] == 0 and b[-1] == total
    sizes = [b[r + 1] - b[r] for r in range(world)]
    assert all(x >= 0 for x in sizes)
    assert max(sizes) - min(sizes) <= 1
    assert b == snplib.snp_shard_plan_sym(m, world)


def test_shard_plan_sym_errors(snplib):
    L = snplib.lib()
    arr = (ctypes.c_int64 * 4)()
    assert L.snp_shard_plan_sym(100, 0, ctypes.cast(arr, ctypes.c_void_p)) == E_RANGE
    assert L.snp_shard_plan_sym(-1, 2, ctypes.cast(arr, ctypes.c_void_p)) == E_RANGE
    assert L.snp_shard_plan_sym(100, 2, None) == E_NULL
    assert L.snp_sym_tiles(-3) == 0


def test_sym_tile_enumeration_is_a_bijection():
    """The row-major upper-triangle order of snp_ld_sym: every (I <= J) exactly once, in
    order, with the closed-form start(I) = I T - I (I - 1) / 2."""
    from paper_conf_ipps_binderlp19_b200.multigpu import sym_tile_coords
    for m in (1, 128, 129, 300, 2048, 5000):
        T = -(-m // 128)
        coords = [sym_tile_coords(m, t) for t in range(T * (T + 1) // 2)]
        assert coords == [(i, j) for i in range(T) for j in range(i, T)]


def test_ld_sym_validation(snplib):
    """snp_ld_sym rejects bad tile ranges and missing outputs before any launch."""
    L = snplib.lib()
    fake = 1 << 20   # an aligned non-NULL address: validation fails before it is touched
    assert L.snp_ld_sym(fake, 300, 8, None, 300, 0, 7, fake, None, None, fake, 4096, None) == E_RANGE
    assert L.snp_ld_sym(fake, 300, 8, None, 300, 3, 2, fake, None, None, fake, 4096, None) == E_RANGE
    assert L.snp_ld_sym(fake, 300, 8, None, 300, -1, 2, fake, None, None, fake, 4096, None) == E_RANGE
    assert L.snp_ld_sym(fake, 300, 8, None, 300, 0, 6, None, None, None, fake, 4096, None) == E_NULL
    assert L.snp_ld_sym(fake, 300, 8, None, 300, 0, 6, None, fake, fake, fake, 4096, None) == E_NULL  # D' needs r2
    assert L.snp_ld_sym(fake, 300, 8, None, 300, 2, 2, fake, None, None, None, 0, None) == OK          # empty range
    assert L.snp_ld_sym(fake + 8, 300, 8, None, 300, 0, 6, fake, None, None, fake, 4096, None) == E_ALIGN
    assert L.snp_sym_unpack(fake, 300, 0, 7, fake, 300, None) == E_RANGE
    assert L.snp_sym_unpack(fake, 300, 0, 6, fake, 299, None) == E_SHAPE
