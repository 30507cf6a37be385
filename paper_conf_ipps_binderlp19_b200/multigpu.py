"""Multi-GPU driver for the SNP-comparison path — one process per GPU.

The path shards with ONE exchange step and no collective inside the hot loop:

* FastID: database rows are sharded (``snp_shard_plan``, 128-row aligned);
  the packed query batch is broadcast from rank 0 (NCCL over NVLink/NVSwitch),
  every rank computes its ``out[nq][nd_r]`` and its per-query best match with
  ``index_base = b_r``; the (count, index) pairs are all-gathered and merged with
  the lowest-global-index tie-break (reading R4).
* LD: output row blocks are sharded; the packed matrix is broadcast from rank 0
  and rank r computes rows ``[b_r, b_{r+1})`` against all columns.
* Symmetric self-LD (f3): the T(T+1)/2 upper-triangle 128 x 128 tiles are split into
  contiguous, equal-count ranges (``snp_shard_plan_sym``); rank r computes its range
  into the packed tile layout of ``snp_ld_sym`` — no tile twice, no mirrored-block
  exchange, balanced within one tile.

The compute callables default to the CUDA library; tests inject oracle-backed
callables to exercise the same exchange logic with the gloo backend on CPU.
The merge is plain tensor plumbing over ``world x nq`` values.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_bounds(rows: int, world: int, align: int = 128) -> list[int]:
    from . import snp_shard_plan
    return snp_shard_plan(rows, world, align)


def merge_best(gc: torch.Tensor, gi: torch.Tensor):
    """gc, gi: [world, nq] per-rank (best count, best global index) -> global best.

    Shards are contiguous and ordered by rank, so among equal counts the lowest
    rank holds the lowest global index; a rank with no rows reports index -1 and
    count 0xFFFFFFFF and never wins unless every rank is empty."""
    c = gc.to(torch.int64) & 0xFFFFFFFF
    idx = gi.to(torch.int64)
    c = torch.where(idx < 0, torch.full_like(c, 1 << 33), c)
    m = c.min(dim=0).values
    first = (c == m).to(torch.int32).argmax(dim=0)        # argmax returns the first maximum
    cols = torch.arange(c.shape[1], device=c.device)
    best_idx = idx[first, cols]
    best_cnt = torch.where(m >= (1 << 33), torch.full_like(m, 0xFFFFFFFF), m)
    return best_cnt, best_idx


KEY_IDX_BITS = 40                     # global database index < 2^40; count < 2^23 above it
KEY_NONE = (1 << 63) - 1              # an empty shard: larger than every real key


def pack_best(bc: torch.Tensor, bi: torch.Tensor, nbits: int | None = None, rows: int | None = None) -> torch.Tensor:
    """(best count, global best index) -> one int64 key ``count << 40 | index`` whose
    minimum over shards is the global best with the lowest-index tie-break (reading R4):
    ONE all-gather and ONE min replace two gathers and an argmin merge.

    A real count must stay below 2^23 (so count << 40 keeps the sign bit clear) and an index
    below 2^40.  Given the shape (nbits bounds every count, rows every global index) the
    bounds are checked on the host; otherwise the values are checked on the device, which
    synchronises the stream (keep that off a timed multi-GPU step)."""
    c = (bc.view(torch.int32) if bc.dtype == torch.uint32 else bc).to(torch.int64) & 0xFFFFFFFF
    if nbits is not None and rows is not None:
        if nbits >= (1 << (63 - KEY_IDX_BITS)):
            raise ValueError("pack_best: nbits >= 2^23: counts do not fit the packed key; use merge_best")
        if rows > (1 << KEY_IDX_BITS):
            raise ValueError("pack_best: more than 2^40 rows do not fit the packed key")
    else:
        real = bi >= 0
        if bool(((c >= (1 << (63 - KEY_IDX_BITS))) & real).any()):
            raise ValueError("pack_best: count >= 2^23 does not fit the packed key; use merge_best")
        if bool((bi >= (1 << KEY_IDX_BITS)).any()):
            raise ValueError("pack_best: index >= 2^40 does not fit the packed key")
    key = (c << KEY_IDX_BITS) | bi.to(torch.int64)
    return torch.where(bi < 0, torch.full_like(key, KEY_NONE), key)


def unpack_best(key: torch.Tensor):
    """Inverse of pack_best; KEY_NONE -> (0xFFFFFFFF, -1)."""
    none = key == KEY_NONE
    c = torch.where(none, torch.full_like(key, 0xFFFFFFFF), key >> KEY_IDX_BITS)
    i = torch.where(none, torch.full_like(key, -1), key & ((1 << KEY_IDX_BITS) - 1))
    return c, i


def gather_best(keys: torch.Tensor, group=None) -> torch.Tensor:
    """keys: [..., nq] local packed keys (any number of ops stacked) -> global minimum over
    the ranks with one all_gather_into_tensor."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world == 1:
        return keys
    g = torch.empty((world,) + tuple(keys.shape), dtype=keys.dtype, device=keys.device)
    dist.all_gather_into_tensor(g.view(-1), keys.contiguous().view(-1), group=group)
    return g.min(dim=0).values


def fastid_step(Q: torch.Tensor, D_shard: torch.Tensor, nbits: int, op: str, index_base: int,
                out: torch.Tensor | None = None, compute=None, best=None, group=None):
    """One sharded FastID step.  Q must be allocated on every rank (its content on
    rank 0 is broadcast).  Returns (local counts, global best count, global best index)."""
    from . import snp_fastid, snp_fastid_best
    compute = compute or (lambda Q_, D_, o_: snp_fastid(Q_, D_, nbits, op, out=o_))
    best = best or (lambda c_, base_: snp_fastid_best(c_, index_base=base_))
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world > 1:
        dist.broadcast(Q.view(torch.int64) if Q.dtype == torch.uint64 else Q, src=0, group=group)
    counts = compute(Q, D_shard, out)
    bc, bi = best(counts, index_base)
    if world == 1:
        return counts, bc.to(torch.int64), bi
    c, i = unpack_best(gather_best(pack_best(bc, bi, nbits=nbits, rows=index_base + D_shard.shape[0]),
                                   group=group))
    return counts, c, i


def ld_step(B: torch.Tensor, nbits: int, lo: int, hi: int, compute=None, group=None):
    """One sharded LD step: broadcast the packed matrix from rank 0, compute rows [lo, hi)."""
    from . import snp_ld_r2
    compute = compute or (lambda A_, B_: snp_ld_r2(A_, B_, nbits, counts=True))
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world > 1:
        dist.broadcast(B.view(torch.int64) if B.dtype == torch.uint64 else B, src=0, group=group)
    return compute(B[lo:hi], B)


def sym_tile_coords(m: int, t: int, tile: int = 128) -> tuple[int, int]:
    """Tile t of the row-major upper triangle (include/snp.h, snp_ld_sym) -> (I, J), I <= J:
    t = start(I) + (J - I), start(I) = I T - I (I - 1) / 2, T = ceil(m / tile)."""
    T = -(-m // tile)
    if not 0 <= t < T * (T + 1) // 2:
        raise ValueError("tile index out of range")
    i = 0
    while i + 1 < T and (i + 1) * T - (i + 1) * i // 2 <= t:
        i += 1
    return i, i + t - (i * T - i * (i - 1) // 2)


def ld_sym_step(B: torch.Tensor, nbits: int, tile_lo: int, tile_hi: int, compute=None, group=None):
    """One sharded symmetric self-LD step: broadcast the packed matrix from rank 0, compute
    this rank's packed-triangle tiles [tile_lo, tile_hi) (snp_shard_plan_sym)."""
    from . import snp_ld_sym
    compute = compute or (lambda B_, lo_, hi_: snp_ld_sym(B_, nbits, lo_, hi_, counts=True))
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world > 1:
        dist.broadcast(B.view(torch.int64) if B.dtype == torch.uint64 else B, src=0, group=group)
    return compute(B, tile_lo, tile_hi)


def ld_sym_step_overlapped(B: torch.Tensor, nbits: int, tile_lo: int, tile_hi: int, block_tiles: int = 16,
                           compute=None, popc=None, group=None):
    """Symmetric self-LD step with the packed-matrix broadcast chunked and overlapped with the
    tiles ("chunk the broadcast into column blocks and overlap it with compute").

    Row blocks of ``block_tiles`` x 128 SNPs are broadcast from rank 0 LAST block first
    (stream.ld_block_plan); tile row I of the packed triangle needs only row blocks >= I, so
    after each block lands this rank computes the part of its range [tile_lo, tile_hi) that
    block completes, while the next block is in flight (NCCL ops are asynchronous on their
    own stream; each compute waits only for the blocks it reads).  Row popcounts of a block
    are counted locally as it lands (``popc(block_rows)``) instead of being broadcast.

    compute(B, lo, hi) -> result for tiles [lo, hi); returns the list of (lo, hi, result)."""
    from .stream import ld_block_plan
    if compute is None:
        from . import snp_ld_sym
        compute = lambda B_, lo_, hi_: snp_ld_sym(B_, nbits, lo_, hi_, counts=True)   # noqa: E731
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    out = []
    for I0, I1, blo, bhi in ld_block_plan(B.shape[0], block_tiles):
        r0, r1 = I0 * 128, min(B.shape[0], I1 * 128)
        if world > 1:
            work = dist.broadcast((B.view(torch.int64) if B.dtype == torch.uint64 else B)[r0:r1], src=0,
                                  group=group, async_op=True)
            work.wait()          # orders this block's consumers after its arrival (stream-ordered on NCCL)
        if popc is not None:
            popc(r0, r1)
        lo, hi = max(tile_lo, blo), min(tile_hi, bhi)
        if lo < hi:
            out.append((lo, hi, compute(B, lo, hi)))
    return out
