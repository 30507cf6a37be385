"""World-size-2 gloo tests (CPU) of the multi-GPU exchange logic.

The compute steps are oracle-backed here (no GPU); what is under test is the
sharding (snp_shard_plan via the C ABI, host-only), the query / matrix broadcast,
the all-gather of per-shard best matches and the lowest-global-index merge.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import snpgen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_ipps_binderlp19_b200 import multigpu

        # ---------------- FastID: DB sharded, queries broadcast, best gathered
        nd, nbits, nq = 700, 300, 9
        db = snpgen.fastid_db(77, np.arange(nd), nbits)
        # plant ties across the shard boundary: rows 100 and 600 identical
        db[600] = db[100]
        b = multigpu.shard_bounds(nd, world, 128)
        lo, hi = b[rank], b[rank + 1]
        Dsh = torch.from_numpy(oracle.pack(db[lo:hi], 6).view(np.int64))
        if rank == 0:
            qg, _ = snpgen.fastid_queries(77, nq, nd, nbits)
            qg[0] = db[100]
            Q = torch.from_numpy(oracle.pack(qg, 6).view(np.int64))
        else:
            Q = torch.zeros((nq, 6), dtype=torch.int64)

        def compute(Q_, D_, out_):
            qq = oracle.unpack(Q_.numpy().view(np.uint64), nbits)
            dd = oracle.unpack(D_.numpy().view(np.uint64), nbits)
            return torch.from_numpy(oracle.counts(qq, dd, "xor").astype(np.int64))

        def best(c_, base_):
            bc, bi = oracle.best(c_.numpy().astype(np.uint32), base_)
            return torch.from_numpy(bc.astype(np.int64)), torch.from_numpy(bi)

        counts, bc, bi = multigpu.fastid_step(Q, Dsh, nbits, "xor", lo, compute=compute, best=best)
        qfull = oracle.unpack(Q.numpy().view(np.uint64), nbits)
        ref_c, ref_i = oracle.best(oracle.counts(qfull, db, "xor"))
        ok_fastid = bool(np.array_equal(bc.numpy(), ref_c.astype(np.int64)) and np.array_equal(bi.numpy(), ref_i))
        ok_tie = int(bi[0]) == 100 and int(bc[0]) == 0
        ok_local = bool(np.array_equal(counts.numpy(), oracle.counts(qfull, db[lo:hi], "xor")))

        # ---------------- LD: packed matrix broadcast, row blocks sharded
        m, nb2 = 300, 130
        g = snpgen.ld_genotypes(78, np.arange(m), nb2, structure=True)
        bb = multigpu.shard_bounds(m, world, 128)
        B = torch.from_numpy(oracle.pack(g, 4).view(np.int64)) if rank == 0 else torch.zeros((m, 4), dtype=torch.int64)

        def ld_compute(A_, B_):
            aa = oracle.unpack(A_.numpy().view(np.uint64), nb2)
            bbm = oracle.unpack(B_.numpy().view(np.uint64), nb2)
            return oracle.ld(aa, bbm)

        r2, dp, nab = multigpu.ld_step(B, nb2, bb[rank], bb[rank + 1], compute=ld_compute)
        r2_ref, _, _ = oracle.ld(g, g)
        ok_ld = bool(np.array_equal(r2, r2_ref[bb[rank]:bb[rank + 1]]))
        q.put((rank, ok_fastid, ok_tie, ok_local, ok_ld, (lo, hi)))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, "error", traceback.format_exc()))


def test_two_rank_gloo_fastid_and_ld():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r in res:
        assert r[1] != "error", r[2]
        rank, ok_fastid, ok_tie, ok_local, ok_ld, rng = r
        assert ok_fastid, f"rank {rank}: merged best != oracle"
        assert ok_tie, f"rank {rank}: tie across shards must go to the lowest global index"
        assert ok_local, f"rank {rank}: local counts wrong for rows {rng}"
        assert ok_ld, f"rank {rank}: LD row block wrong"


def test_merge_best_edge_cases():
    from paper_conf_ipps_binderlp19_b200.multigpu import merge_best
    gc = torch.tensor([[5, 3, 0xFFFFFFFF], [3, 3, 7]], dtype=torch.int64)
    gi = torch.tensor([[10, 11, -1], [200, 201, 202]], dtype=torch.int64)
    c, i = merge_best(gc, gi)
    assert c.tolist() == [3, 3, 7]
    assert i.tolist() == [200, 11, 202]
    c, i = merge_best(torch.tensor([[0xFFFFFFFF]]), torch.tensor([[-1]]))
    assert c.tolist() == [0xFFFFFFFF] and i.tolist() == [-1]


def test_stream_chunk_plan():
    """f2 host logic: contiguous, ordered, 128-aligned chunks covering [0, nd)."""
    from paper_conf_ipps_binderlp19_b200.stream import chunk_plan
    assert chunk_plan(0, 1000) == []
    assert chunk_plan(100, 1000) == [(0, 100)]
    assert chunk_plan(1000, 300) == [(0, 256), (256, 512), (512, 768), (768, 1000)]
    assert chunk_plan(1000, 5) == [(r, min(1000, r + 128)) for r in range(0, 1000, 128)]
    for nd, ch in [(1, 1), (12345, 4096), (4096, 4096)]:
        p = chunk_plan(nd, ch)
        assert p[0][0] == 0 and p[-1][1] == nd
        assert all(a[1] == b[0] for a, b in zip(p, p[1:]))
        assert all(r0 % 128 == 0 for r0, _ in p)


def test_pack_best_keys():
    """Packed (count << 40 | index) keys: min == lowest count, then lowest index; empty
    shards never win; round trip."""
    from paper_conf_ipps_binderlp19_b200.multigpu import pack_best, unpack_best
    bc = torch.tensor([[5, 3, 0xFFFFFFFF, 4], [3, 3, 7, 4]], dtype=torch.int64)
    bi = torch.tensor([[10, 11, -1, (1 << 39) + 5], [200, 201, 202, 6]], dtype=torch.int64)
    k = pack_best(bc, bi)
    c, i = unpack_best(k.min(dim=0).values)
    assert c.tolist() == [3, 3, 7, 4] and i.tolist() == [200, 11, 202, 6]
    c, i = unpack_best(pack_best(torch.tensor([0xFFFFFFFF]), torch.tensor([-1])))
    assert c.tolist() == [0xFFFFFFFF] and i.tolist() == [-1]
    u = torch.tensor([0x7FFFFF, 0], dtype=torch.int32).view(torch.uint32)   # uint32 counts
    c, i = unpack_best(pack_best(u, torch.tensor([3, 4])))
    assert c.tolist() == [0x7FFFFF, 0] and i.tolist() == [3, 4]


def test_pack_best_rejects_counts_that_overflow_the_key():
    """count << 40 must keep the sign bit clear: counts >= 2^23 (possible for profiles of
    more than 2^23 SNPs) are rejected instead of silently winning the min as negatives."""
    from paper_conf_ipps_binderlp19_b200.multigpu import pack_best
    with pytest.raises(ValueError):
        pack_best(torch.tensor([1 << 23]), torch.tensor([0]))
    with pytest.raises(ValueError):
        pack_best(torch.tensor([1]), torch.tensor([1 << 40]))
    # shape-bounded form (no device sync): the host check rejects the shape instead
    with pytest.raises(ValueError):
        pack_best(torch.tensor([1]), torch.tensor([0]), nbits=1 << 23, rows=10)
    with pytest.raises(ValueError):
        pack_best(torch.tensor([1]), torch.tensor([0]), nbits=100, rows=(1 << 40) + 1)
    k = pack_best(torch.tensor([5, 0xFFFFFFFF]), torch.tensor([7, -1]), nbits=100, rows=10)
    assert k.tolist() == [(5 << 40) | 7, (1 << 63) - 1]
    pack_best(torch.tensor([(1 << 23) - 1, 0xFFFFFFFF]), torch.tensor([0, -1]))   # empty shard is fine


def _sym_worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_ipps_binderlp19_b200 import multigpu, snp_shard_plan_sym
        m, nbits = 300, 130
        g = snpgen.ld_genotypes(79, np.arange(m), nbits, structure=True)
        B = torch.from_numpy(oracle.pack(g, 4).view(np.int64)) if rank == 0 else torch.zeros((m, 4), dtype=torch.int64)
        b = snp_shard_plan_sym(m, world)
        lo, hi = b[rank], b[rank + 1]

        def tiles_compute(B_, lo_, hi_):
            # oracle-backed tiles in the packed layout: tile u = block (I, J), zeros past m
            gg = oracle.unpack(B_.numpy().view(np.uint64), nbits)
            out = np.zeros((hi_ - lo_, 128, 128), dtype=np.float64)
            for u, t in enumerate(range(lo_, hi_)):
                I, J = multigpu.sym_tile_coords(m, t)
                r2, _, _ = oracle.ld(gg[128 * I:128 * I + 128], gg[128 * J:128 * J + 128])
                out[u, :r2.shape[0], :r2.shape[1]] = r2
            return out

        mine = multigpu.ld_sym_step(B, nbits, lo, hi, compute=tiles_compute)
        got = [None] * world
        dist.all_gather_object(got, (lo, hi, mine))
        full = np.full((m, m), np.nan)
        seen = set()
        for lo_, hi_, tl in got:
            for u, t in enumerate(range(lo_, hi_)):
                assert t not in seen
                seen.add(t)
                I, J = multigpu.sym_tile_coords(m, t)
                blk = tl[u][:min(128, m - 128 * I), :min(128, m - 128 * J)]
                full[128 * I:128 * I + blk.shape[0], 128 * J:128 * J + blk.shape[1]] = blk
                full[128 * J:128 * J + blk.shape[1], 128 * I:128 * I + blk.shape[0]] = blk.T
        r2_ref, _, _ = oracle.ld(g, g)
        q.put((rank, bool(np.array_equal(full, r2_ref)), len(seen), hi - lo))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, "error", traceback.format_exc()))


def test_two_rank_gloo_symmetric_ld_plan():
    """f3 + e: the triangle-balanced plan over 2 ranks — each rank computes only its tile
    range (oracle-backed tiles in the packed layout); together the ranks cover every upper-
    triangle tile once and the mirrored union equals the oracle's full r2 matrix."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sym_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r in res:
        assert r[1] != "error", r[2]
        rank, ok, nseen, mine = r
        assert ok, f"rank {rank}: reconstructed symmetric matrix != oracle"
        assert nseen == 6                      # T = 3 tiles per side: 6 upper-triangle tiles
        assert mine == 3                       # balanced: 3 + 3


@pytest.mark.parametrize("m,bt", [(1, 1), (128, 4), (700, 2), (2048, 16), (32768, 16), (5000, 3)])
def test_stream_ld_block_plan(m, bt):
    """f2 for LD host logic: blocks streamed last-first; together their tile ranges cover
    every packed-triangle tile exactly once, in contiguous pieces; every tile of a block's
    range needs only rows of that block or of blocks streamed before it."""
    from paper_conf_ipps_binderlp19_b200.multigpu import sym_tile_coords
    from paper_conf_ipps_binderlp19_b200.stream import ld_block_plan
    T = -(-m // 128)
    plan = ld_block_plan(m, bt)
    assert [p[0] for p in plan] == sorted([p[0] for p in plan], reverse=True)
    covered = sorted((lo, hi) for _, _, lo, hi in plan)
    assert covered[0][0] == 0 and covered[-1][1] == T * (T + 1) // 2
    assert all(a[1] == b[0] for a, b in zip(covered, covered[1:]))
    arrived_from = T
    for I0, I1, lo, hi in plan:
        arrived_from = I0                      # rows >= 128 * I0 are on the device now
        for t in ([lo, hi - 1] if hi - lo > 2 else range(lo, hi)):
            I, J = sym_tile_coords(m, t)
            assert I0 <= I < I1 and J >= arrived_from


def _sym_overlap_worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_ipps_binderlp19_b200 import multigpu, snp_shard_plan_sym
        m, nbits = 700, 130
        g = snpgen.ld_genotypes(80, np.arange(m), nbits, structure=True)
        B = torch.from_numpy(oracle.pack(g, 4).view(np.int64)) if rank == 0 else torch.zeros((m, 4), dtype=torch.int64)
        b = snp_shard_plan_sym(m, world)
        lo, hi = b[rank], b[rank + 1]
        seen_rows = []

        def tiles_compute(B_, lo_, hi_):
            gg = oracle.unpack(B_.numpy().view(np.uint64), nbits)
            res = {}
            for t in range(lo_, hi_):
                I, J = multigpu.sym_tile_coords(m, t)
                # every row this tile reads must have arrived already
                assert all(min(seen_rows) <= 128 * x for x in (I, J))
                res[t] = oracle.ld(gg[128 * I:128 * I + 128], gg[128 * J:128 * J + 128])[2]
            return res

        parts = multigpu.ld_sym_step_overlapped(B, nbits, lo, hi, block_tiles=2, compute=tiles_compute,
                                                popc=lambda r0, r1: seen_rows.append(r0))
        mine = {}
        for plo, phi, res in parts:
            assert lo <= plo < phi <= hi
            mine.update(res)
        got = [None] * world
        dist.all_gather_object(got, mine)
        full = np.full((m, m), -1, dtype=np.int64)
        for d in got:
            for t, blk in d.items():
                I, J = multigpu.sym_tile_coords(m, t)
                full[128 * I:128 * I + blk.shape[0], 128 * J:128 * J + blk.shape[1]] = blk
                full[128 * J:128 * J + blk.shape[1], 128 * I:128 * I + blk.shape[0]] = blk.T
        _, _, n_ref = oracle.ld(g, g)
        q.put((rank, bool(np.array_equal(full, n_ref)), sorted(mine) == list(range(lo, hi))))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, "error", traceback.format_exc()))


def test_two_rank_gloo_symmetric_ld_overlapped_broadcast():
    """e + f3: the packed matrix broadcast in row blocks (last first) overlapped with the
    tiles each block completes; every rank computes exactly its tile range, no tile reads a
    row that has not arrived, and the union equals the oracle's full count matrix."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sym_overlap_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r in res:
        assert r[1] != "error", r[2]
        assert r[1] and r[2], r
