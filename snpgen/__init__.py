"""Seeded synthetic genotype generator shared by tests, smoke() and bench.py.

This module holds NONE of the method's arithmetic (no packing, no popcount,
no comparison).  It only draws 0/1 genotype bytes from a counter-based hash so
that any row can be regenerated independently, bit-identically, on the host
(numpy) and on a device (torch), e.g. to feed sampled rows to the CPU oracle
while the GPU packs the full matrix.

Recipe (after SURVEY §8d):
  * per-SNP minor-allele frequency f ~ U[0.05, 0.5), stored as an integer
    32-bit threshold T (f = T / 2^32);
  * genotype bit (row r, column k) = H(seed, r, k) < T[snp], where snp = r for
    LD matrices (rows are SNPs over samples, P:L107 / Fig. 2) and snp = k for
    FastID profiles (rows are profiles over SNPs);
  * optional LD structure rows: row 0 all-zero, row 1 all-one, every 64th row a
    copy of its predecessor, every 97th row the complement of its own draw
    (exercises r2 in {0, 1}, D' = +-1 and the monomorphic 0/0 case);
  * FastID queries: the first half are copies of random database rows with 0-8
    random flips (identity search), the second half are the OR of three
    database rows (mixtures).

H is a 32-bit integer mixer evaluated in int64 arithmetic with every product
< 2^63, so numpy and torch produce identical bits.
"""
from __future__ import annotations

import numpy as np

_M32 = 0xFFFFFFFF
_C1 = 0x7FEB352D
_C2 = 0x2C1B3C6D
_SALT_ROW = 0x1B873593
_SALT_MAF = 0x5BD1E995 & 0x7FFFFFFF
_SALT_Q = 0x68E31DA4
_SALT_FLIP = 0x3C6EF372
_SALT_NFLIP = 0x27D4EB2F
_SALT_MIX = 0x165667B1

F_LO = 214748365          # 0.05 * 2^32 (rounded up)
F_SPAN = 1932735283       # 0.45 * 2^32


def _mix(x):
    """32-bit avalanche mixer on int64 arrays/tensors holding values < 2^32."""
    x = x ^ (x >> 16)
    x = (x * _C1) & _M32
    x = x ^ (x >> 15)
    x = (x * _C2) & _M32
    x = x ^ (x >> 16)
    return x


def _h(seed: int, salt: int, a):
    """H(seed, salt, a) for an int64 array a of non-negative values < 2^32."""
    s = _mix_scalar(((seed & _M32) ^ salt) & _M32)
    return _mix(a ^ s)


def _mix_scalar(v: int) -> int:
    return int(_mix(np.array([v], dtype=np.int64))[0])


def _row_keys(seed: int, rows):
    return _h(seed, _SALT_ROW, rows)


def maf_thresholds(seed: int, idx):
    """Integer thresholds T (f = T/2^32, f in [0.05, 0.5)) for SNP indices idx."""
    return F_LO + _h(seed, _SALT_MAF, idx) % F_SPAN


# ---------------------------------------------------------------- backends

def _np_arange(n, device=None):
    return np.arange(n, dtype=np.int64)


def _np_asarray(a, device=None):
    return np.asarray(a, dtype=np.int64)


def _torch_mod():
    import torch
    return torch


def _raw_bits(seed: int, rows, nbits: int, orient: str, xp: str, device=None):
    """uint8 [len(rows)][nbits] drawn from H; rows is an int64 array/tensor."""
    if xp == "numpy":
        cols = np.arange(nbits, dtype=np.int64)
        rk = _row_keys(seed, rows)[:, None]
        h = _mix(rk ^ cols[None, :])
        if orient == "ld":
            thr = maf_thresholds(seed, rows)[:, None]
        else:
            thr = maf_thresholds(seed, cols)[None, :]
        return (h < thr).astype(np.uint8)
    torch = _torch_mod()
    cols = torch.arange(nbits, dtype=torch.int64, device=device)
    rk = _row_keys(seed, rows)[:, None]
    h = _mix(rk ^ cols[None, :])
    if orient == "ld":
        thr = maf_thresholds(seed, rows)[:, None]
    else:
        thr = maf_thresholds(seed, cols)[None, :]
    return (h < thr).to(torch.uint8)


def _as_rows(rows, xp, device):
    if xp == "numpy":
        return np.asarray(rows, dtype=np.int64)
    torch = _torch_mod()
    return torch.as_tensor(rows, dtype=torch.int64, device=device)


def ld_genotypes(seed: int, rows, nbits: int, structure: bool = False,
                 xp: str = "numpy", device=None):
    """LD matrix rows (SNPs x samples) as uint8 0/1, for the given row indices."""
    rows = _as_rows(rows, xp, device)
    if not structure:
        return _raw_bits(seed, rows, nbits, "ld", xp, device)
    # structure: r%64==0 (r>=64) copies row r-1; then r==0 zeros, r==1 ones,
    # r%97==0 complements its own draw.  Resolve the copy first (one level).
    src = rows.clone() if xp != "numpy" else rows.copy()
    dup = (rows % 64 == 0) & (rows >= 64)
    src[dup] = rows[dup] - 1
    g = _raw_bits(seed, src, nbits, "ld", xp, device)
    comp = (src % 97 == 0) & (src > 1)
    g[comp] = 1 - g[comp]
    g[src == 0] = 0
    g[src == 1] = 1
    return g


def fastid_db(seed: int, rows, nbits: int, xp: str = "numpy", device=None):
    """FastID database profiles (profiles x SNPs) as uint8 0/1."""
    return _raw_bits(seed, _as_rows(rows, xp, device), nbits, "fastid", xp, device)


def fastid_query_plan(seed: int, nq: int, nd: int, nbits: int):
    """Host-side plan of the planted queries: list of (kind, db_rows, flip_cols).

    kind 'copy'  : query = db row with the listed columns flipped (<= 8 flips)
    kind 'mix'   : query = OR of the listed db rows
    """
    q = np.arange(nq, dtype=np.int64)
    plan = []
    for i in range(nq):
        if i < (nq + 1) // 2:
            j = int(_h(seed, _SALT_Q, q[i:i + 1])[0]) % nd
            nflip = int(_h(seed, _SALT_NFLIP, q[i:i + 1])[0]) % 9
            ks = np.arange(nflip, dtype=np.int64) + 16 * i
            flips = sorted(set(int(v) % nbits for v in _h(seed, _SALT_FLIP, ks)))
            plan.append(("copy", [j], flips))
        else:
            ks = np.arange(3, dtype=np.int64) + 4 * i
            js = [int(v) % nd for v in _h(seed, _SALT_MIX, ks)]
            plan.append(("mix", js, []))
    return plan


def fastid_queries(seed: int, nq: int, nd: int, nbits: int, xp: str = "numpy", device=None):
    """Planted queries (uint8 0/1 [nq][nbits]) and their plan."""
    plan = fastid_query_plan(seed, nq, nd, nbits)
    out = []
    for kind, js, flips in plan:
        g = fastid_db(seed, js, nbits, xp, device)
        if kind == "copy":
            row = g[0].clone() if xp != "numpy" else g[0].copy()
            for k in flips:
                row[k] = 1 - row[k]
        else:
            row = g.max(0) if xp == "numpy" else g.amax(0)
        out.append(row)
    if xp == "numpy":
        q = np.stack(out) if out else np.zeros((0, nbits), np.uint8)
    else:
        torch = _torch_mod()
        q = torch.stack(out) if out else torch.zeros((0, nbits), dtype=torch.uint8, device=device)
    return q, plan


def random_bytes_nonzero(shape, seed: int):
    """Random non-zero byte values (to test 'non-zero = minor allele')."""
    rng = np.random.default_rng(seed)
    return rng.integers(1, 256, size=shape, dtype=np.uint8)
