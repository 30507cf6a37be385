"""f2 — end-to-end streaming FastID search.

The paper measures FastID end to end, with the database moved to the device in chunks and
the transfers overlapped with the comparisons by double buffering.  Here the
packed database stays in pinned host memory and is streamed through two device buffers:
the H2D copy of chunk k+1 runs on a copy stream (copy engine) while chunk k is searched on
the compute stream (``snp_fastid_search``, per-query best match, no count matrix), events
order buffer reuse.  Each chunk's best (count, global index) lands in its own row of a
``[chunks, nq]`` table; chunks are contiguous and increasing, so the final merge is the
multi-GPU merge with the lowest-global-index tie-break (reading R4).

Host logic only (chunk planning, stream/event ordering, argument marshalling): every
comparison runs in the library's kernels.
"""
from __future__ import annotations

import torch


def chunk_plan(nd: int, chunk_rows: int, align: int = 128) -> list[tuple[int, int]]:
    """Contiguous [r0, r1) database chunks of at most chunk_rows rows (a multiple of
    align, at least align); the last one is ragged.  nd = 0 gives no chunks."""
    if nd < 0 or chunk_rows < 1 or align < 1:
        raise ValueError("nd >= 0, chunk_rows >= 1, align >= 1")
    step = max(align, chunk_rows // align * align)
    return [(r0, min(nd, r0 + step)) for r0 in range(0, nd, step)]


def stream_search(Q: torch.Tensor, D_host: torch.Tensor, nbits: int, ops=("xor", "andnot"),
                  popD_host: torch.Tensor | None = None, chunk_rows: int = 1 << 20,
                  index_base: int = 0):
    """Per-query best match of every op over a database in pinned host memory.

    Q: packed queries on the device; D_host: packed database rows (uint64, pinned CPU);
    popD_host: optional pinned uint32 row popcounts (else counted on the device per
    chunk).  Returns a list (one per op) of (best_count uint32-in-int64, best_index int64)
    device tensors of length nq; an empty database gives (0xFFFFFFFF, -1)."""
    from . import snp_fastid_search, snp_fastid_search_workspace_bytes, snp_row_popc
    from .multigpu import merge_best
    if isinstance(ops, str):
        ops = (ops,)
    if D_host.is_cuda or not D_host.is_pinned():
        raise ValueError("D_host must be a pinned CPU tensor")
    if popD_host is not None and (popD_host.is_cuda or not popD_host.is_pinned()):
        raise ValueError("popD_host must be a pinned CPU tensor")
    dev = Q.device
    nq, nd = Q.shape[0], D_host.shape[0]
    plan = chunk_plan(nd, chunk_rows)
    nops = len(ops)
    bc = torch.full((nops, max(1, len(plan)), nq), 0xFFFFFFFF, dtype=torch.int64, device=dev)
    bi = torch.full((nops, max(1, len(plan)), nq), -1, dtype=torch.int64, device=dev)
    if not plan:
        return [(bc[j, 0], bi[j, 0]) for j in range(nops)]
    rows_max = max(r1 - r0 for r0, r1 in plan)
    nbuf = min(2, len(plan))
    Dbuf = [torch.empty((rows_max, D_host.shape[1]), dtype=D_host.dtype, device=dev) for _ in range(nbuf)]
    Pbuf = [torch.empty(rows_max, dtype=torch.uint32, device=dev) for _ in range(nbuf)] if popD_host is not None else None
    # per-chunk results are written as uint32 counts / int64 indices, then widened
    cnt32 = torch.empty((nops, len(plan), nq), dtype=torch.uint32, device=dev)
    # the dispatcher's kernel choice (and so its scratch) depends on the chunk's row count: a
    # ragged last chunk with few rows can take a path that needs more workspace than a full
    # chunk, so size for every distinct chunk length
    ws_need = max(snp_fastid_search_workspace_bytes(nq, rows, nbits, nops) for rows in {r1 - r0 for r0, r1 in plan})
    ws = torch.zeros(max(1, ws_need), dtype=torch.uint8, device=dev)   # zero-filled once (snp.h)
    comp = torch.cuda.current_stream(dev)
    copy = torch.cuda.Stream(dev)
    copy.wait_stream(comp)   # the buffers (and Q) were just allocated / produced on comp
    copied = [torch.cuda.Event() for _ in range(nbuf)]
    freed = [torch.cuda.Event() for _ in range(nbuf)]
    for k, (r0, r1) in enumerate(plan):
        b, rows = k % nbuf, r1 - r0
        with torch.cuda.stream(copy):
            if k >= nbuf:
                copy.wait_event(freed[b])          # chunk k - nbuf is done with buffer b
            Dbuf[b][:rows].copy_(D_host[r0:r1], non_blocking=True)
            if Pbuf is not None:
                Pbuf[b][:rows].copy_(popD_host[r0:r1], non_blocking=True)
            copied[b].record(copy)
        comp.wait_event(copied[b])
        D = Dbuf[b][:rows]
        pd = Pbuf[b][:rows] if Pbuf is not None else snp_row_popc(D, nbits)
        snp_fastid_search(Q, D, nbits, ops, counts=False,
                          best=[(cnt32[j, k], bi[j, k]) for j in range(nops)],
                          index_base=index_base + r0, ws=ws, popD=pd)
        freed[b].record(comp)
    for buf in Dbuf + (Pbuf or []):
        buf.record_stream(copy)
    bc[:, :len(plan)] = cnt32.view(torch.int32).to(torch.int64) & 0xFFFFFFFF
    return [merge_best(bc[j], bi[j]) for j in range(nops)]


def ld_block_plan(m: int, block_tiles: int) -> list[tuple[int, int, int, int]]:
    """Row blocks of block_tiles tile rows in the order they are streamed (last first), each
    with the packed-triangle tile range it completes: (I0, I1, tile_lo, tile_hi).  Tile row I
    holds tiles (I, J), J >= I, so it needs only row blocks >= I — all of which arrive no
    later than block I (host logic, covered by tests on CPU)."""
    T = -(-m // 128)

    def start(I):      # first tile of tile row I (row-major upper triangle)
        return I * T - I * (I - 1) // 2
    return [(b0, min(T, b0 + block_tiles), start(b0), start(min(T, b0 + block_tiles)))
            for b0 in range(0, T, block_tiles)][::-1]


def stream_ld_sym(A_host: torch.Tensor, nbits: int, block_tiles: int = 16, r2: bool = True, counts: bool = True,
                  dprime: bool = False, out_host: dict | None = None, device=None):
    """f2 for LD — end-to-end symmetric self-LD from a packed matrix in pinned host memory
    (the paper's end-to-end mode, §VI.A: input and output transfers double-buffered
    and overlapped with the kernels; Fig. 6).

    Row blocks of ``block_tiles`` x 128 SNPs are copied host -> device on a copy stream in
    REVERSE order; tile row I of the packed upper triangle (``snp_ld_sym``) needs only row
    blocks >= I, so as soon as block b has arrived (all later ones arrived before it) its
    tile rows are computed on the compute stream while block b - 1 is in flight.  Row
    popcounts are counted per block as it lands.  With ``out_host`` (dict of pinned host
    tensors 'r2' / 'counts' / 'dprime' shaped like the device outputs) each block's tiles are
    copied back on a second copy stream while the next block computes.

    Returns dict of device outputs ([snp_sym_tiles(m)][128][128]) and the device matrix."""
    from . import snp_ld_sym, snp_row_popc, snp_sym_tiles
    if A_host.is_cuda or not A_host.is_pinned():
        raise ValueError("A_host must be a pinned CPU tensor")
    if block_tiles < 1:
        raise ValueError("block_tiles >= 1")
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    m = A_host.shape[0]
    T = -(-m // 128)
    ntot = snp_sym_tiles(m)
    A = torch.empty(A_host.shape, dtype=A_host.dtype, device=dev)
    pop = torch.empty(m, dtype=torch.uint32, device=dev)
    outs = {}
    if r2:
        outs["r2"] = torch.empty((ntot, 128, 128), dtype=torch.float32, device=dev)
    if dprime:
        outs["dprime"] = torch.empty((ntot, 128, 128), dtype=torch.float32, device=dev)
    if counts:
        outs["counts"] = torch.empty((ntot, 128, 128), dtype=torch.uint32, device=dev)
    if not outs:
        raise ValueError("nothing requested")
    comp = torch.cuda.current_stream(dev)
    h2d, d2h = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    h2d.wait_stream(comp)
    d2h.wait_stream(comp)

    plan = ld_block_plan(m, block_tiles)
    blocks = [(I0, I1) for I0, I1, _, _ in plan]
    arrived = []
    for I0, I1 in blocks:                       # all H2D copies queued up front, last block first
        r0, r1 = I0 * 128, min(m, I1 * 128)
        with torch.cuda.stream(h2d):
            A[r0:r1].copy_(A_host[r0:r1], non_blocking=True)
            ev = torch.cuda.Event()
            ev.record(h2d)
        arrived.append(ev)
    for (I0, I1, lo, hi), ev in zip(plan, arrived):
        r0, r1 = I0 * 128, min(m, I1 * 128)
        comp.wait_event(ev)
        snp_row_popc(A[r0:r1], nbits, out=pop[r0:r1])
        snp_ld_sym(A, nbits, lo, hi, popA=pop, r2=outs.get("r2", False)[lo:hi] if r2 else False,
                   dprime=outs["dprime"][lo:hi] if dprime else None,
                   counts=outs["counts"][lo:hi] if counts else None)
        if out_host is not None:
            done = torch.cuda.Event()
            done.record(comp)
            d2h.wait_event(done)
            with torch.cuda.stream(d2h):
                for k, t in outs.items():
                    if k in out_host:
                        out_host[k][lo:hi].copy_(t[lo:hi], non_blocking=True)
    comp.wait_stream(d2h)
    comp.wait_stream(h2d)
    for t in [A, pop, *outs.values()]:
        t.record_stream(h2d)
        t.record_stream(d2h)
    return outs, A
