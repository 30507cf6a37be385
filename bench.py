#!/usr/bin/env python
"""bench.py — SNP comparisons/s on B200 (BASELINE.json metric), one JSON line.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload fastid1m|ld2k|ld32k|fastid20m]
                    [--impl ours|reference]

A *step* is one pass of the whole hot path over one batch:
  fastid*: a1 pack the query batch -> (N>1: NCCL broadcast of the packed queries)
           -> a3+a4+a6 ONE snp_fastid_search pass over the resident packed database
           giving XOR (identity search, Eq. 2) and ANDNOT (mixture analysis, Eq. 3)
           count matrices and the best match per query for both (N>1: all-gather of
           the per-shard bests).  --fastid-step separate runs snp_fastid +
           snp_fastid_best per op instead (two database passes + two count re-reads).
  ld*:     a1 pack the genotype matrix -> (N>1: NCCL broadcast of the packed
           matrix) -> a2 row popcounts + a3 AND-count GEMM + a5 r2 epilogue
           (counts and r2 written) for this rank's row block.
value = SNP comparisons (bit pairs, M*N*nbits per op) of all ranks / max-over-ranks
device time.  Inputs live in HBM before the timed region (the database is larger
than L2; for the LD workloads L2 is flushed before every timed step and the flushes'
own time, measured by a graph of the flushes alone, is subtracted).  At N = 1 the
timed steps are one CUDA-graph replay with events on the stream around it (no event
nodes inside the graph).  `e2e` repeats the measurement through the public API with
pinned host inputs (H2D of the genotype bytes) and a D2H of each step's result
(FastID at N = 1: double-buffered on a copy stream, overlapped with the next step).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # BASELINE.json configs; fastid1m = configs[1] (the N=1 headline), ld2k = configs[0]
    "fastid1m": dict(kind="fastid", nq=64, nd=1_000_000, nbits=4096, scaling="weak", seed=1002,
                     desc="FastID 64 queries x 1,000,000 profiles x 4,096 SNPs, XOR + ANDNOT (configs[1])"),
    "fastid20m": dict(kind="fastid", nq=1024, nd=20_000_000, nbits=8192, scaling="strong", seed=1004,
                      desc="FastID 1,024 queries x 20,000,000 profiles x 8,192 SNPs (configs[3])"),
    "ld2k": dict(kind="ld", m=2048, nbits=4096, scaling="strong", seed=1001,
                 desc="LD 2,048 x 2,048 SNPs x 4,096 samples, counts + r2 (configs[0])"),
    "ld32k": dict(kind="ld", m=32768, nbits=16384, scaling="strong", seed=1003,
                  desc="LD 32,768 x 32,768 SNPs x 16,384 samples, counts + r2 (configs[2])"),
}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=None)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--workload", default="fastid1m", choices=sorted(WORKLOADS))
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--variant", default="auto", choices=["auto", "popc", "tc"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-graph", dest="graph", action="store_false",
                   help="run the timed steps eagerly instead of replaying a captured CUDA graph")
    p.add_argument("--fastid-step", default="fused", choices=["fused", "separate"],
                   help="fused: one snp_fastid_search pass for XOR+ANDNOT counts and best matches; "
                        "separate: snp_fastid + snp_fastid_best per op")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="target oracle CPU time")
    p.add_argument("--ld-layout", default="tri", choices=["tri", "rows"],
                   help="tri: f3 packed upper-triangle tiles, triangle-balanced over ranks (snp_ld_sym); "
                        "rows: full m x m matrix, output row blocks per rank (snp_ld_r2)")
    a = p.parse_args()
    if a.warmup < 3:
        a.warmup = 3
    return a


# ----------------------------------------------------------------------------- peaks

def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    src = "measured"
    try:
        with open(path) as f:
            pk = json.load(f)
    except Exception:
        pk = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
              "sm_max_mhz": 1965.0}
        src = "fallback (B200_PROFILING.md)"
    sm_mhz = float(pk.get("sm_max_mhz", 1965.0))
    # POPC issue rate per SM, measured with the paper's §V.D throughput microbenchmark
    # (tools/alu_probe.cu; profiles/round2/alu_probe.txt): 15.98 / clk / SM
    popc_clk, popc_src = 16.0, "assumed 16 POPC/clk/SM"
    try:
        with open(os.path.join(ROOT, "profiles", "alu_peaks.json")) as f:
            popc_clk = float(json.load(f)["popc_per_clk_sm"])
            popc_src = "measured POPC/clk/SM (tools/alu_probe.cu, profiles/alu_peaks.json)"
    except Exception:
        pass
    return {
        "src": src,
        "hbm_gbs": float(pk["hbm_gbs"]),
        # POPC pipe: 148 SMs x 16 POPC/clk/SM x 32 bits x max SM clock (P:L281 convention),
        # in TOPS-equivalent (2 ops per bit comparison) — DESIGN.md §6.
        "popc_tops": 2 * 148 * popc_clk * 32 * sm_mhz * 1e6 / 1e12,
        "popc_src": popc_src, "popc_per_clk_sm": popc_clk,
        # int8 tensor: measured bf16 dense x nominal i8:bf16 ratio 2 (4.5 vs 2.25 PF spec).
        "i8_tops": 2.0 * float(pk["bf16_tflops"]),
        # fp4 (kind::mxf4) tensor: measured bf16 dense x nominal fp4:bf16 ratio 4 (9 vs 2.25 PF).
        "f4_tops": 4.0 * float(pk["bf16_tflops"]),
        "i8_tops_sustained": 2.0 * float(pk.get("bf16_tflops_sustained", pk["bf16_tflops"])),
        "sm_max_mhz": sm_mhz,
    }


# ----------------------------------------------------------------------------- clocks

class ClockSampler:
    """Samples SM clock and throttle reasons with NVML every ~5 ms while running."""
    BAD = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
           "hw_power_brake_slowdown": 0x80}
    NAMES = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
             0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
             0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
             0x100: "display_clock_setting"}

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.reasons = 0
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["nvml-unavailable"]}
        reasons = [n for b, n in self.NAMES.items() if self.reasons & b and b != 0x1]
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(self.samples)}


# ----------------------------------------------------------------------------- dist

def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import torch
    local = local % max(1, torch.cuda.device_count())   # (several ranks per GPU only in logic tests)
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")   # gloo: multi-rank logic test on 1 GPU
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    return rank, world, local


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(world):
    import torch
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize()


# ----------------------------------------------------------------------------- CPU oracle

def cpu_baseline(wl, seconds, cores=None):
    """Time the oracle (as it stands) on a bounded sample of the workload."""
    import numpy as np

    import oracle
    import snpgen
    oracle.build()
    cores = cores or os.cpu_count()
    if wl["kind"] == "fastid":
        nq, nbits = wl["nq"], wl["nbits"]
        q, _ = snpgen.fastid_queries(wl["seed"], nq, wl["nd"], nbits)
        probe = 64
        db = snpgen.fastid_db(wl["seed"], np.arange(probe), nbits)
        t0 = time.perf_counter()
        oracle.counts(q, db, "xor")
        dt = time.perf_counter() - t0
        rows = max(probe, int(probe * seconds / 2 / max(dt, 1e-6)))
        db = snpgen.fastid_db(wl["seed"], np.arange(rows), nbits)
        t0 = time.perf_counter()
        for op in ("xor", "andnot"):
            oracle.counts(q, db, op)
        dt = time.perf_counter() - t0
        cmp = 2 * nq * rows * nbits
        sample = f"{nq} queries x {rows} database rows x {nbits} SNPs, ops xor+andnot (full workload: {wl['nd']} rows)"
    else:
        m, nbits = wl["m"], wl["nbits"]
        gall = np.concatenate([snpgen.ld_genotypes(wl["seed"], np.arange(r0, min(m, r0 + 2048)), nbits,
                                                   structure=True) for r0 in range(0, m, 2048)])
        t0 = time.perf_counter()
        oracle.ld(gall[:8], gall)
        dt = time.perf_counter() - t0
        rows = max(8, min(m, int(8 * seconds / max(dt, 1e-6))))
        t0 = time.perf_counter()
        oracle.ld(gall[:rows], gall)
        dt = time.perf_counter() - t0
        cmp = rows * m * nbits
        sample = f"{rows} SNP rows x {m} SNPs x {nbits} samples, counts + r2 + D' (full workload: {m} rows)"
    full = (2 * wl["nq"] * wl["nd"] * wl["nbits"]) if wl["kind"] == "fastid" else wl["m"] * wl["m"] * wl["nbits"]
    return {"value": cmp / dt, "unit": "comparisons/s", "cores": cores, "kind": "oracle",
            "sample": sample, "seconds": round(dt, 3),
            "extrapolated": cmp < full, "full_workload_seconds_extrapolated": round(full / (cmp / dt), 1),
            "protocol": "profiles/round2/oracle_protocol.json (full cfg-1 / cfg-2 runs, 1-thread cfg-1)",
            "host": host_popcount_peak(cores)}


def host_popcount_peak(cores):
    """The host's theoretical popcount throughput as the paper states it for CPUs
    (cores x clock x bits per cycle): 64 bits/cycle/core with POPCNT, 512 with
    AVX-512 VPOPCNTDQ.  Context for the oracle number, not a target."""
    model, mhz, flags = "?", None, ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                k, _, v = line.partition(":")
                k = k.strip()
                if k == "model name" and model == "?":
                    model = v.strip()
                elif k == "cpu MHz" and mhz is None:
                    mhz = float(v)
                elif k == "flags" and not flags:
                    flags = v
    except OSError:
        pass
    try:
        with open("/sys/devices/system/cpu/cpu0/cpufreq/cpuinfo_max_freq") as f:
            mhz = int(f.read()) / 1e3
    except (OSError, ValueError):
        pass
    bits = 512 if "avx512_vpopcntdq" in flags.split() else 64
    peak = cores * (mhz or 0) * 1e6 * bits
    return {"model": model, "mhz": mhz, "popcount_bits_per_cycle": bits,
            "theoretical_cmp_per_s": peak, "oracle_note": "the oracle is plain bit-by-bit C (not tuned)"}


# ----------------------------------------------------------------------------- workloads

FASTID_STEP = "fused"

def _gen_fastid_db(snp, snpgen, torch, seed, row0, rows, nbits, dev, chunk=32768):
    D = torch.empty((rows, snp.snp_words(nbits)), dtype=torch.uint64, device=dev)
    for r0 in range(0, rows, chunk):
        r1 = min(rows, r0 + chunk)
        g = snpgen.fastid_db(seed, torch.arange(row0 + r0, row0 + r1, device=dev), nbits,
                             xp="torch", device=dev)
        snp.snp_pack(g, out=D[r0:r1])
        del g
    return D


def setup_fastid(wl, rank, world, dev):
    import numpy as np
    import torch

    import paper_conf_ipps_binderlp19_b200 as snp
    import snpgen
    nq, nbits = wl["nq"], wl["nbits"]
    if wl["scaling"] == "weak":
        nd_total = wl["nd"] * world
        lo, hi = rank * wl["nd"], (rank + 1) * wl["nd"]
    else:
        nd_total = wl["nd"]
        b = snp.snp_shard_plan(nd_total, world, 128)
        lo, hi = b[rank], b[rank + 1]
    nd = hi - lo
    D = _gen_fastid_db(snp, snpgen, torch, wl["seed"], lo, nd, nbits, dev)
    # the database's row popcounts are prepared once with it (a static forensic database,
    # SURVEY §8d), outside the timed step; the search reads them instead of re-counting
    popD = snp.snp_row_popc(D, nbits)
    q, _ = snpgen.fastid_queries(wl["seed"], nq, nd_total, nbits)
    qbytes = torch.from_numpy(np.ascontiguousarray(q)).to(dev)
    qhost = torch.from_numpy(np.ascontiguousarray(q)).pin_memory()
    Q = torch.empty((nq, snp.snp_words(nbits)), dtype=torch.uint64, device=dev)
    OPS = ("xor", "andnot")
    fused = FASTID_STEP == "fused"
    outs = {op: torch.empty((nq, nd), dtype=torch.uint32, device=dev) for op in OPS}
    best = {op: (torch.empty(nq, dtype=torch.uint32, device=dev), torch.empty(nq, dtype=torch.int64, device=dev))
            for op in OPS}
    if fused:
        ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, len(OPS)), dtype=torch.uint8,
                         device=dev)
    else:
        ws = {op: (torch.empty(snp.snp_fastid_workspace_bytes(nq, nd, nbits, op), dtype=torch.uint8, device=dev))
              for op in OPS}
    merged = {}
    res_host = {op: (torch.empty(nq, dtype=torch.uint32).pin_memory(), torch.empty(nq, dtype=torch.int64).pin_memory())
                for op in OPS}
    keys_host = torch.empty((len(OPS), nq), dtype=torch.int64).pin_memory() if world > 1 else None
    # full e2e (N=1): the count matrices themselves copied back to pinned host memory
    full_host = ({op: torch.empty((nq, nd), dtype=torch.uint32).pin_memory() for op in OPS}
                 if world == 1 and nq * nd * 4 * len(OPS) <= (1 << 30) else None)
    st = dict(D=D, Q=Q, qbytes=qbytes, qhost=qhost, outs=outs, best=best, ws=ws, lo=lo, nd=nd,
              res_host=res_host)
    cmp_rank = 2 * nq * nd * nbits
    cmp_all = 2 * nq * (nd_total if wl["scaling"] == "strong" else wl["nd"] * world) * nbits

    def _search():
        # a3 + a4 + a6 for both ops in ONE pass over the resident database (f1)
        snp.snp_fastid_search(Q, D, nbits, OPS, counts=[outs[op] for op in OPS],
                              best=[best[op] for op in OPS], index_base=lo, ws=ws, popD=popD)

    def _fast(op):
        return lambda: snp.snp_fastid(Q, D, nbits, op, out=outs[op], popD=popD,
                                      ws=ws[op] if ws[op].numel() else None)

    def _best(op):
        return lambda: snp.snp_fastid_best(outs[op], index_base=lo, best_count=best[op][0], best_index=best[op][1])

    # e2e at N = 1, pipelined as the paper's host framework double-buffers its transfers
    # (P:L269): the query bytes of step i+1 go up and the best matches of step i come down on a
    # copy stream while step i searches; query and result buffers are double-buffered (events
    # guard both hazards).  Every step still moves its own inputs H2D and its result D2H.
    pipe = None
    if world == 1 and fused:
        rb = 2 * nq * 8 + 2 * nq * 4                       # int64 [2][nq] indices, uint32 [2][nq] counts
        dres = [torch.empty(rb, dtype=torch.uint8, device=dev) for _ in range(2)]
        pipe = dict(
            i=0, primed=False, copy=torch.cuda.Stream(dev),
            q=[qbytes, torch.empty_like(qbytes)],
            dres=dres,
            hres=[torch.empty(rb, dtype=torch.uint8).pin_memory() for _ in range(2)],
            best=[[(d[16 * nq:].view(torch.uint32).view(2, nq)[j], d[:16 * nq].view(torch.int64).view(2, nq)[j])
                   for j in range(len(OPS))] for d in dres],
            copied=[torch.cuda.Event() for _ in range(2)], packed=[torch.cuda.Event() for _ in range(2)],
            searched=[torch.cuda.Event() for _ in range(2)], fetched=[torch.cuda.Event() for _ in range(2)],
            used=[False, False])

    def e2e_step():
        s = torch.cuda.current_stream()
        c = pipe["copy"]
        i = pipe["i"]
        b, nb = i % 2, (i + 1) % 2
        if not pipe["primed"]:
            with torch.cuda.stream(c):
                c.wait_stream(s)
                pipe["q"][b].copy_(qhost, non_blocking=True)       # this step's queries H2D
                pipe["copied"][b].record(c)
            pipe["primed"] = True
        s.wait_event(pipe["copied"][b])
        snp.snp_pack(pipe["q"][b], nbits=nbits, out=Q)              # a1
        pipe["packed"][b].record(s)
        with torch.cuda.stream(c):   # the next step's queries go up while this step searches
            c.wait_event(pipe["packed"][nb] if pipe["used"][nb] else pipe["packed"][b])
            pipe["q"][nb].copy_(qhost, non_blocking=True)
            pipe["copied"][nb].record(c)
        if pipe["used"][b]:
            s.wait_event(pipe["fetched"][b])                       # the D2H of step i-2 has read it
        snp.snp_fastid_search(Q, D, nbits, OPS, counts=[outs[op] for op in OPS], best=pipe["best"][b],
                              index_base=lo, ws=ws, popD=popD)     # a3 + a4 + a6
        pipe["searched"][b].record(s)
        with torch.cuda.stream(c):   # this step's best matches come down behind the next H2D
            c.wait_event(pipe["searched"][b])
            pipe["hres"][b].copy_(pipe["dres"][b], non_blocking=True)
            pipe["fetched"][b].record(c)
        pipe["used"][b] = True
        pipe["i"] = i + 1

    def e2e_check():
        """The pipelined e2e's last result on the host equals the device-resident step's best."""
        if pipe is None or pipe["i"] == 0:
            return None
        torch.cuda.synchronize()
        b = (pipe["i"] - 1) % 2
        h = pipe["hres"][b]
        hi = h[:16 * nq].view(torch.int64).view(2, nq)
        hc = h[16 * nq:].view(torch.uint32).view(2, nq)
        return all(torch.equal(hi[j], best[op][1].cpu()) and torch.equal(hc[j], best[op][0].cpu())
                   for j, op in enumerate(OPS))

    def step(kev=None, host=False):
        s = torch.cuda.current_stream()
        if host is True and pipe is not None:
            e2e_step()
            return
        if host:   # e2e: H2D of this step's query genotype bytes
            qbytes.copy_(qhost, non_blocking=True)
        if rank == 0:
            snp.snp_pack(qbytes, nbits=nbits, out=Q)                       # a1
        if world > 1:
            import torch.distributed as dist
            dist.broadcast(Q.view(torch.int64), src=0)                     # queries -> all ranks
        if fused:
            if kev is not None:
                kev[0].record(s)
            _search()
            if kev is not None:
                kev[1].record(s)
        else:   # one snp_fastid + snp_fastid_best per op (two database passes)
            for i, op in enumerate(OPS):
                if kev is not None:
                    kev[2 * i].record(s)
                _fast(op)()                                                # a3+a4
                if kev is not None:
                    kev[2 * i + 1].record(s)
                _best(op)()                                                # a6
        if world > 1:
            # global best per query and op, lowest global index on ties: both
            # ops' (count, index) packed into int64 keys, ONE all-gather, ONE min
            from paper_conf_ipps_binderlp19_b200 import multigpu
            # bounds checked on the host from the shape (no device sync inside the timed step)
            keys = torch.stack([multigpu.pack_best(*best[op], nbits=nbits, rows=nd_total) for op in OPS])
            merged["keys"] = multigpu.gather_best(keys)
            if host:   # e2e: D2H of the step's result, the GLOBAL best (count << 40 | index keys)
                keys_host.copy_(merged["keys"], non_blocking=True)
            return
        for op in OPS:
            bc, bi = best[op]
            if host:   # e2e: D2H of the step's result (per-query best count and index)
                res_host[op][0].copy_(bc, non_blocking=True)
                res_host[op][1].copy_(bi, non_blocking=True)
            if host == "full":   # full e2e: the count matrices too
                full_host[op].copy_(outs[op], non_blocking=True)

    # the same device-resident step as separately capturable parts (N=1 graph mode)
    pack_part = (lambda: snp.snp_pack(qbytes, nbits=nbits, out=Q), False)
    if fused:
        parts = [pack_part, (_search, True)]
    else:
        parts = [pack_part, (_fast("xor"), True), (_best("xor"), False), (_fast("andnot"), True),
                 (_best("andnot"), False)]

    # algorithmic bytes of the dominant kernel per launch: DB + queries read, counts written
    words = (nbits + 63) // 64
    nout = len(OPS) if fused else 1
    alg_bytes = (nd + nq) * words * 8 + nout * nq * nd * 4
    return dict(step=step, parts=parts, cmp_rank=cmp_rank, cmp_all=cmp_all,
                kernel_launches_per_step=1 if fused else 2, step_mode=FASTID_STEP,
                kernel_cmp=nq * nd * nbits, kernel_bytes=alg_bytes,
                h2d=nq * nbits, d2h=(2 * nq * 8 if world > 1 else 2 * nq * 12), l2_flush=False,
                d2h_full=(len(OPS) * nq * nd * 4 if full_host is not None else None),
                e2e_check=e2e_check,
                e2e_launch=("eager public-API calls per step (no graph); the query H2D of step i+1 and the result "
                            "D2H of step i run on a copy stream while step i searches (double-buffered, P:L269)"
                            if pipe is not None else "eager public-API calls per step (no graph)"),
                e2e_result=("global best (count, index) per query for XOR and ANDNOT (merged over ranks); "
                            "the count matrices stay sharded in HBM" if world > 1 else
                            "per-query best (count, index) for XOR and ANDNOT; the two nq x nd count matrices "
                            "stay in HBM (e2e_full copies them back too)"),
                l2_note=f"inputs larger than L2 ({nd * snp.snp_words(nbits) * 8 / 1e6:.0f} MB database per rank)",
                state=st, snp=snp)


LD_LAYOUT = "tri"


def setup_ld(wl, rank, world, dev):
    if LD_LAYOUT == "tri":
        return setup_ld_tri(wl, rank, world, dev)
    import torch

    import paper_conf_ipps_binderlp19_b200 as snp
    import snpgen
    m, nbits = wl["m"], wl["nbits"]
    b = snp.snp_shard_plan(m, world, 128)
    lo, hi = b[rank], b[rank + 1]
    rows = hi - lo
    words = snp.snp_words(nbits)
    # genotype bytes resident in HBM (rank 0 holds the full matrix and packs it)
    G = None
    if rank == 0:
        G = torch.empty((m, nbits), dtype=torch.uint8, device=dev)
        for r0 in range(0, m, 2048):
            r1 = min(m, r0 + 2048)
            G[r0:r1] = snpgen.ld_genotypes(wl["seed"], torch.arange(r0, r1, device=dev), nbits,
                                           structure=True, xp="torch", device=dev)
    Ghost = G.cpu().pin_memory() if (rank == 0) else None
    B = torch.empty((m, words), dtype=torch.uint64, device=dev)
    pop = torch.empty(m, dtype=torch.uint32, device=dev)
    r2 = torch.empty((rows, m), dtype=torch.float32, device=dev)
    cnt = torch.empty((rows, m), dtype=torch.uint32, device=dev)
    ws = torch.empty(max(1, snp.snp_ld_workspace_bytes(rows, m, nbits)), dtype=torch.uint8, device=dev)
    res_host = torch.empty(1, dtype=torch.float32).pin_memory()
    full_host = ((torch.empty((rows, m), dtype=torch.float32).pin_memory(),
                  torch.empty((rows, m), dtype=torch.uint32).pin_memory()) if rows * m * 8 <= (1 << 30) else None)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def step(kev=None, host=False):
        s = torch.cuda.current_stream()
        if rank == 0:
            if host:
                G.copy_(Ghost, non_blocking=True)                           # e2e H2D
            snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop)             # a1 + a2
        if world > 1:
            import torch.distributed as dist
            dist.broadcast(B.view(torch.int64), src=0)
            dist.broadcast(pop.view(torch.int32), src=0)
        if kev is not None:
            kev[0].record(s)
        snp.snp_ld_r2(B[lo:hi], B, nbits, popA=pop[lo:hi], popB=pop, r2=r2, counts=cnt, ws=ws)   # a3 + a5
        if kev is not None:
            kev[1].record(s)
        if host:   # e2e: D2H of the step's result statistic (r2 of the first pair)
            res_host.copy_(r2.view(-1)[:1], non_blocking=True)
        if host == "full":   # full e2e: the r2 and count matrices of this rank
            full_host[0].copy_(r2, non_blocking=True)
            full_host[1].copy_(cnt, non_blocking=True)

    def l2flush():
        flush.add_(1)

    parts = [(lambda: snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop), False),
             (lambda: snp.snp_ld_r2(B[lo:hi], B, nbits, popA=pop[lo:hi], popB=pop, r2=r2, counts=cnt, ws=ws), True)] \
        if rank == 0 else None

    alg_bytes = (rows + m) * words * 8 + rows * m * 8
    return dict(step=step, parts=parts, cmp_rank=rows * m * nbits, cmp_all=m * m * nbits, kernel_launches_per_step=1,
                kernel_cmp=rows * m * nbits, kernel_bytes=alg_bytes, h2d=(m * nbits if rank == 0 else 0),
                d2h=4, l2_flush=True, flush=l2flush, d2h_full=(rows * m * 8 if full_host is not None else None),
                e2e_result="r2 of the first pair (the r2 and count matrices stay in HBM; e2e_full copies them back)",
                l2_note="L2 flushed (256 MB read+write) before every timed step; the flushes timed alone and subtracted",
                state=dict(B=B, r2=r2, cnt=cnt), snp=snp)


def setup_ld_tri(wl, rank, world, dev):
    """LD as symmetric self-LD in the packed upper-triangle tile layout (f3): rank r computes
    the contiguous tile range of snp_shard_plan_sym (balanced within one tile, no tile twice,
    no mirrored-block exchange); counts + r2 per tile."""
    import torch

    import paper_conf_ipps_binderlp19_b200 as snp
    import snpgen
    m, nbits = wl["m"], wl["nbits"]
    b = snp.snp_shard_plan_sym(m, world)
    lo, hi = b[rank], b[rank + 1]
    nt = hi - lo
    words = snp.snp_words(nbits)
    G = None
    if rank == 0:
        G = torch.empty((m, nbits), dtype=torch.uint8, device=dev)
        for r0 in range(0, m, 2048):
            r1 = min(m, r0 + 2048)
            G[r0:r1] = snpgen.ld_genotypes(wl["seed"], torch.arange(r0, r1, device=dev), nbits,
                                           structure=True, xp="torch", device=dev)
    Ghost = G.cpu().pin_memory() if (rank == 0) else None
    B = torch.empty((m, words), dtype=torch.uint64, device=dev)
    pop = torch.empty(m, dtype=torch.uint32, device=dev)
    r2 = torch.empty((max(nt, 1), 128, 128), dtype=torch.float32, device=dev)
    cnt = torch.empty((max(nt, 1), 128, 128), dtype=torch.uint32, device=dev)
    res_host = torch.empty(1, dtype=torch.float32).pin_memory()
    out_bytes = nt * 128 * 128 * 8
    full_host = ((torch.empty(r2.shape, dtype=torch.float32).pin_memory(),
                  torch.empty(cnt.shape, dtype=torch.uint32).pin_memory()) if out_bytes <= (1 << 30) else None)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    ldws = torch.empty(max(1, snp.snp_ld_sym_workspace_bytes(m, nbits)), dtype=torch.uint8, device=dev)

    def compute():
        snp.snp_ld_sym(B, nbits, lo, hi, popA=pop, r2=r2, counts=cnt, ws=ldws)  # a3 + a5 (f3 tiles)

    # end to end at N = 1 (the paper's mode): the matrix packed on the host (as the
    # paper's CPU packer leaves it) in pinned memory, streamed in row blocks overlapped with
    # the tiles (stream.stream_ld_sym); e2e_full also copies every tile back, block by block
    from paper_conf_ipps_binderlp19_b200.stream import stream_ld_sym
    Bhost = None
    if world == 1:
        snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop)
        Bhost = B.cpu().pin_memory()
    host_tiles = ({"r2": full_host[0], "counts": full_host[1]} if full_host is not None else None)

    def step(kev=None, host=False):
        s = torch.cuda.current_stream()
        if host and world == 1:
            outs, _ = stream_ld_sym(Bhost, nbits, block_tiles=16,
                                    out_host=host_tiles if host == "full" else None)
            res_host.copy_(outs["r2"].view(-1)[:1], non_blocking=True)
            return
        if rank == 0:
            if host:
                G.copy_(Ghost, non_blocking=True)                           # e2e H2D
            snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop)             # a1 + a2
        if kev is not None:
            kev[0].record(s)
        if world > 1:
            # packed matrix broadcast in row blocks (last first), each rank's tiles computed as
            # the blocks they read land (SURVEY §8e overlap); popcounts counted per block
            from paper_conf_ipps_binderlp19_b200 import multigpu
            multigpu.ld_sym_step_overlapped(
                B, nbits, lo, hi, block_tiles=16,
                compute=lambda B_, a, b_: snp.snp_ld_sym(B_, nbits, a, b_, popA=pop, r2=r2[a - lo:b_ - lo],
                                                         counts=cnt[a - lo:b_ - lo]),
                popc=(None if rank == 0 else lambda r0, r1: snp.snp_row_popc(B[r0:r1], nbits, out=pop[r0:r1])))
        else:
            compute()
        if kev is not None:
            kev[1].record(s)
        if host:   # e2e: D2H of the step's result statistic (r2 of the first pair)
            res_host.copy_(r2.view(-1)[:1], non_blocking=True)
        if host == "full":   # full e2e: this rank's r2 and count tiles
            full_host[0].copy_(r2, non_blocking=True)
            full_host[1].copy_(cnt, non_blocking=True)

    def l2flush():
        flush.add_(1)

    parts = [(lambda: snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop), False), (compute, True)] \
        if rank == 0 else None
    alg_bytes = m * words * 8 + out_bytes
    return dict(step=step, parts=parts, cmp_rank=nt * 128 * 128 * nbits, cmp_all=m * m * nbits,
                kernel_launches_per_step=1, kernel_cmp=nt * 128 * 128 * nbits, kernel_bytes=alg_bytes,
                h2d=(m * words * 8 if world == 1 else (m * nbits if rank == 0 else 0)), d2h=4, l2_flush=True,
                flush=l2flush, d2h_full=(out_bytes if full_host is not None else None),
                e2e_result=("host-packed matrix (pinned) streamed in 2048-row blocks overlapped with the tiles "
                            "(stream_ld_sym, P:L269); result = r2 of the first pair, the tiles stay in HBM "
                            "(e2e_full copies every tile back block by block)" if world == 1 else
                            "genotype bytes H2D on rank 0, packed and broadcast; r2 of the first pair"),
                layout=f"packed upper triangle: tiles [{lo}, {hi}) of {b[-1]} (128 x 128, row-major triangle order)",
                l2_note="L2 flushed (256 MB read+write) before every timed step; the flushes timed alone and subtracted",
                state=dict(B=B, r2=r2, cnt=cnt), snp=snp)


# ----------------------------------------------------------------------------- main timing

def timed(wlrun, steps, host, world, kernel_events=True, graph=None):
    """Time `steps` steps; returns (total_ms max over ranks, per-kernel mean ms).

    With `graph` (a captured CUDA graph of one step, N=1) each step is one graph
    replay, so the device time excludes Python/launch overhead; the per-kernel
    events were captured inside the graph.  Without it the step runs eagerly."""
    import torch
    s = torch.cuda.current_stream()
    nk = 2 * wlrun["kernel_launches_per_step"]
    kevs = [[torch.cuda.Event(enable_timing=True) for _ in range(nk)] for _ in range(steps)]
    sev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]

    def one(i):
        if graph is not None:
            j = 0
            for g, is_kernel in graph["parts"]:
                if is_kernel and kernel_events:
                    kevs[i][j].record(s)
                g.replay()
                if is_kernel and kernel_events:
                    kevs[i][j + 1].record(s)
                    j += 2
        else:
            wlrun["step"](kevs[i] if kernel_events else None, host)

    barrier(world)
    if wlrun["l2_flush"]:
        for i in range(steps):
            wlrun["flush"]()
            sev[i][0].record(s)
            one(i)
            sev[i][1].record(s)
    else:
        sev[0][0].record(s)
        for i in range(steps):
            one(i)
        sev[-1][1].record(s)
    torch.cuda.synchronize()
    barrier(world)
    if wlrun["l2_flush"]:
        total = sum(a.elapsed_time(b) for a, b in sev)
    else:
        total = sev[0][0].elapsed_time(sev[-1][1])
    kms = []
    if kernel_events:
        for ev in kevs:
            for j in range(0, nk, 2):
                kms.append(ev[j].elapsed_time(ev[j + 1]))
    total = max_over_ranks(total, world)
    return total, (statistics.mean(kms) if kms else None)


def capture_run(wlrun, steps, mode="step"):
    """Capture ALL timed steps in one CUDA graph with NO timing nodes inside it: an event-record
    node between kernels costs ~4-5 us and breaks their programmatic-dependent-launch overlap
    (scripts/step_overhead.py: FastID-1M step 174.4 us bare, 183.2 us with step-boundary event
    nodes, 196.5 us with event nodes around the search call too), so timing events are recorded
    on the stream around the replay instead.  mode "step": every part of the step (the L2 flush
    before each step where the workload asks for it); "kernel": only the dominant kernel's call
    (after the same flush); "flush": the flushes alone (subtracted from the other two)."""
    import torch

    import paper_conf_ipps_binderlp19_b200 as snp
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        for fn, _ in wlrun["parts"]:
            fn()                                   # warm the capture stream
    torch.cuda.current_stream().wait_stream(side)
    torch.cuda.synchronize()
    n0 = snp.snp_launch_count()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for i in range(steps):
            if wlrun["l2_flush"]:
                wlrun["flush"]()
            for fn, is_kernel in wlrun["parts"]:
                if mode == "step" or (mode == "kernel" and is_kernel):
                    fn()
    torch.cuda.synchronize()
    return {"graph": g, "launches": snp.snp_launch_count() - n0}


def replay_ms(run, world):
    """One replay of a captured graph, CUDA events on the stream around it (max over ranks)."""
    import torch
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier(world)
    torch.cuda.synchronize()
    e0.record(s)
    run["graph"].replay()
    e1.record(s)
    torch.cuda.synchronize()
    barrier(world)
    return max_over_ranks(e0.elapsed_time(e1), world)


def run_ours(args):
    import torch

    rank, world, local = dist_setup(args)
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    wl = WORKLOADS[args.workload]
    peaks = load_peaks()
    import paper_conf_ipps_binderlp19_b200 as snp
    snp.snp_set_variant(args.variant)
    steps = args.steps or (200 if wl["kind"] == "fastid" else 20)
    global FASTID_STEP, LD_LAYOUT
    FASTID_STEP = args.fastid_step
    LD_LAYOUT = args.ld_layout
    wlrun = (setup_fastid if wl["kind"] == "fastid" else setup_ld)(wl, rank, world, dev)
    torch.cuda.synchronize()

    for _ in range(args.warmup):
        wlrun["step"](None, False)
    torch.cuda.synchronize()
    graph = None
    use_graph = args.graph and world == 1 and wlrun.get("parts") is not None
    n0 = snp.snp_launch_count()
    if use_graph:
        # the whole timed region (all steps) as one captured graph with events only at step
        # boundaries; one untimed replay first.  The dominant kernel's launch durations come
        # from a second replay of the same steps with event-record nodes around that kernel
        # (event nodes between kernels break their programmatic-dependent-launch overlap, so
        # they stay out of the step timing)
        graph = capture_run(wlrun, steps, "step")
        kgraph = capture_run(wlrun, steps, "kernel")
        fgraph = capture_run(wlrun, steps, "flush") if wlrun["l2_flush"] else None
        for r in (graph, kgraph, fgraph):
            if r is not None:
                r["graph"].replay()               # one untimed replay each
        torch.cuda.synchronize()
        with ClockSampler(local) as clk:
            step_all = replay_ms(graph, world)
            kern_all = replay_ms(kgraph, world)
            flush_all = replay_ms(fgraph, world) if fgraph is not None else 0.0
        # steps (or dominant-kernel calls) back to back, the flushes' own time subtracted
        total_ms = step_all - flush_all
        kern_ms = (kern_all - flush_all) / steps
        launches = graph["launches"]             # kernels replayed from the graph (all steps)
    else:
        with ClockSampler(local) as clk:
            total_ms, kern_ms = timed(wlrun, steps, False, world, graph=None)
        launches = snp.snp_launch_count() - n0
    variant = snp.snp_last_variant()
    kernel = snp.snp_last_kernel()
    ms = total_ms / steps
    value = wlrun["cmp_all"] / (ms / 1e3)

    e2e = None
    if not args.no_e2e:
        for _ in range(2):
            wlrun["step"](None, True)
        torch.cuda.synchronize()
        e2e_ms, _ = timed(wlrun, steps, True, world, kernel_events=False)
        e2e = {"value": wlrun["cmp_all"] / (e2e_ms / steps / 1e3), "unit": "comparisons/s",
               "h2d_bytes_per_step": wlrun["h2d"], "d2h_bytes_per_step": wlrun["d2h"],
               "ms_per_step": e2e_ms / steps, "result": wlrun["e2e_result"],
               "launch": wlrun.get("e2e_launch", "eager public-API calls per step (no graph)")}
        if wlrun.get("e2e_check") is not None:
            e2e["result_matches_device_step"] = wlrun["e2e_check"]()
        if world == 1 and wlrun.get("d2h_full"):
            # the same step with every output matrix copied back to the host (PCIe-bound)
            fsteps = max(3, min(steps, 10))
            wlrun["step"](None, "full")
            torch.cuda.synchronize()
            f_ms, _ = timed(wlrun, fsteps, "full", world, kernel_events=False)
            e2e["full"] = {"value": wlrun["cmp_all"] / (f_ms / fsteps / 1e3), "unit": "comparisons/s",
                           "h2d_bytes_per_step": wlrun["h2d"], "d2h_bytes_per_step": wlrun["d2h_full"],
                           "ms_per_step": f_ms / fsteps, "steps": fsteps}

    # roofline of the dominant kernel (the bit-GEMM launch), live CUDA-event durations
    kcmp = wlrun["kernel_cmp"]
    kcmp_eff = kcmp
    if wl["kind"] == "ld" and LD_LAYOUT == "tri":
        # executed work is the rank's tiles (kernel_cmp); the effective rate counts the
        # m * m * nbits comparisons of the full symmetric matrix those tiles represent
        kcmp_eff = wlrun["cmp_all"] // world
    elif kernel in ("tc_mxf4_sym", "tc_mxf4_sym_pair"):
        # f3 symmetric self-LD executes only the upper-triangle 128 x 128 tiles (SURVEY §8d:
        # roofline on the executed work, M*N*nbits reported as the effective rate)
        T = -(-wl["m"] // 128)
        kcmp = T * (T + 1) // 2 * 128 * 128 * wl["nbits"]
    tops = 2 * kcmp / (kern_ms / 1e3) / 1e12
    if kernel in ("tc_mxf4", "tc_mxf4_sym", "tc_mxf4_sym_pair", "tc_mxf4_pair", "fastid_mxf4"):
        roof = {"bound": "tensor", "achieved": tops, "peak": peaks["f4_tops"], "unit": "TOPS",
                "peak_src": f"fp4 dense = 4 x bf16 burst ({peaks['src']} MEASURED_PEAKS.json)"}
    elif kernel == "tc_i8":
        roof = {"bound": "tensor", "achieved": tops, "peak": peaks["i8_tops"], "unit": "TOPS",
                "peak_src": f"int8 dense = 2 x bf16 burst ({peaks['src']} MEASURED_PEAKS.json)"}
    else:
        roof = {"bound": "alu", "achieved": tops, "peak": peaks["popc_tops"], "unit": "TOPS",
                "peak_src": f"POPC pipe: 148 SM x {peaks['popc_per_clk_sm']:.2f}/clk x 32 bit x "
                            f"{peaks['sm_max_mhz']:.0f} MHz ({peaks['popc_src']})"}
    roof["frac"] = roof["achieved"] / roof["peak"]
    roof["kernel_ms"] = kern_ms
    roof["kernel"] = kernel
    traffic = None   # dram bytes read+write per launch from one ncu --set full capture (profiles/)
    prof = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                traffic = json.load(f).get(f"{args.workload}:{kernel}")
        except Exception:
            traffic = None
    hbm_gbs = wlrun["kernel_bytes"] / (kern_ms / 1e3) / 1e9
    roof_hbm = {"bound": "hbm", "achieved": hbm_gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": hbm_gbs / peaks["hbm_gbs"], "alg_bytes_per_launch": wlrun["kernel_bytes"],
                "kernel_ms": kern_ms, "kernel": kernel, "peak_src": f"{peaks['src']} MEASURED_PEAKS.json copy"}
    roof["traffic"] = roof_hbm["traffic"] = traffic
    roof["alg_cmp_per_launch"] = kcmp
    if kcmp != kcmp_eff:
        roof["effective_cmp_per_launch"] = kcmp_eff
        roof["effective_tops"] = 2 * kcmp_eff / (kern_ms / 1e3) / 1e12
    # the binding roof of this launch: its algorithmic bytes at the HBM peak vs its
    # comparisons at the pipe's peak (FastID at 64 queries is HBM-bound, LD and FastID
    # with 1,024 queries are compute-bound; north_star)
    t_hbm = wlrun["kernel_bytes"] / (peaks["hbm_gbs"] * 1e9)
    t_pipe = 2 * kcmp / (roof["peak"] * 1e12)
    if t_hbm >= t_pipe:
        roof_primary, roof_secondary = roof_hbm, roof
    else:
        roof_primary, roof_secondary = roof, roof_hbm

    out = None
    if rank == 0:
        out = {
            "metric": "SNP comparisons/sec",
            "value": value, "unit": "comparisons/s",
            "n_gpus": world, "steps": steps, "warmup": args.warmup,
            "ms_per_step": ms, "higher_is_better": True,
            "scaling": wl["scaling"], "vs_baseline": None,
            "dtype": "u1 (bit-packed u64 words; uint32 counts, fp32 r2)",
            "data": "synthetic (seeded counter-based genotype generator, MAF ~ U[0.05,0.5))",
            "config": {"workload": args.workload, "desc": wl["desc"],
                       **{k: v for k, v in wl.items() if k in ("nq", "nd", "m", "nbits")},
                       "variant": variant, "kernel": kernel, "l2": wlrun["l2_note"],
                       **({"step": wlrun["step_mode"]} if "step_mode" in wlrun else {}),
                       "launch": (("one captured CUDA graph of all timed steps, CUDA events around its replay"
                                   + ("; the L2 flush before every step timed alone (a graph of the flushes) "
                                      "and subtracted" if wlrun["l2_flush"] else ""))
                                  if use_graph else "eager"),
                       **({"kernel_timing": "dominant kernel's call replayed back to back (same flushes, "
                                            "subtracted), CUDA events around the replay"} if use_graph else {}),
                       **({"output": wlrun["layout"]} if "layout" in wlrun else {}),
                       "parallelism": (f"db-shard x{world}" if wl["kind"] == "fastid" else
                                       f"triangle-tile-shard x{world}" if LD_LAYOUT == "tri" else
                                       f"row-shard x{world}")},
            "word_ops_per_s": value / 64, "tops_eq": 2 * value / 1e12,
            "roofline": roof_primary, "roofline_secondary": roof_secondary,
            "gpu_launches": launches,
            "clocks": clk.summary(),
            "e2e": e2e,
        }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(wl, args.cpu_seconds)
        out["gpu_over_cpu"] = value / out["cpu_baseline"]["value"]
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


def run_reference(args):
    """Reference arm = the CPU oracle (this tier has no reference implementation)."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if rank != 0:
        return
    wl = WORKLOADS[args.workload]
    steps = args.steps or 3
    per_step = max(1.0, min(args.cpu_seconds, 60.0 / (steps + args.warmup)))
    for _ in range(args.warmup):
        cpu_baseline(wl, per_step / 4)
    runs = [cpu_baseline(wl, per_step) for _ in range(steps)]
    value = statistics.median(r["value"] for r in runs)
    cb = dict(runs[-1])
    cb["value"] = value
    out = {
        "impl": "reference", "metric": "SNP comparisons/sec", "value": value, "unit": "comparisons/s",
        "n_gpus": world, "steps": steps, "warmup": args.warmup,
        "ms_per_step": statistics.median(r["seconds"] for r in runs) * 1e3,
        "higher_is_better": True, "scaling": wl["scaling"], "vs_baseline": None,
        "dtype": "u1 (unpacked bytes, bit-by-bit)", "data": "synthetic",
        "config": {"workload": args.workload, "desc": wl["desc"],
                   **{k: v for k, v in wl.items() if k in ("nq", "nd", "m", "nbits")}},
        "cpu_baseline": cb,
        "e2e": {"value": value, "unit": "comparisons/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
