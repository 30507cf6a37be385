"""SURVEY §8d oracle-timing protocol on the host cores (a reported baseline, not a target):
full oracle runs on configs[0] (LD-2K) with all cores and with ONE thread, a full run on
configs[1] (FastID-1M, XOR + ANDNOT), and seeded row samples of configs[2] (LD-32K) and
configs[3] (FastID-20M) timed and extrapolated linearly (labelled "extrapolated").  The
host's theoretical popcount peak is printed the way the paper states CPU peaks.

Each measurement runs in a subprocess so OMP_NUM_THREADS takes effect; the oracle is used
as it stands (never tuned).  Output: one JSON object (stdout), e.g. into
profiles/round2/oracle_protocol.json."""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import json, sys, time
sys.path.insert(0, ROOT)
import numpy as np
import oracle, snpgen
kind, seed, rows, n, nbits, nq = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5]), int(sys.argv[6])
if kind == "ld":
    g = np.concatenate([snpgen.ld_genotypes(seed, np.arange(r0, min(n, r0 + 2048)), nbits, structure=True)
                        for r0 in range(0, n, 2048)])
    t0 = time.perf_counter(); oracle.ld(g[:rows], g); dt = time.perf_counter() - t0
    cmp = rows * n * nbits
else:
    q, _ = snpgen.fastid_queries(seed, nq, n, nbits)
    db = snpgen.fastid_db(seed, np.arange(rows), nbits)
    t0 = time.perf_counter()
    for op in ("xor", "andnot"):
        oracle.counts(q, db, op)
    dt = time.perf_counter() - t0
    cmp = 2 * nq * rows * nbits
print(json.dumps({"seconds": dt, "cmp": cmp}))
'''.replace("ROOT", repr(ROOT))


def run(kind, seed, rows, n, nbits, nq=0, threads=None):
    env = dict(os.environ)
    if threads:
        env["OMP_NUM_THREADS"] = str(threads)
    out = subprocess.run([sys.executable, "-c", CHILD, kind, str(seed), str(rows), str(n), str(nbits), str(nq)],
                         env=env, capture_output=True, text=True, check=True).stdout
    return json.loads(out.strip().splitlines()[-1])


def main():
    sys.path.insert(0, ROOT)
    import oracle
    oracle.build()
    from bench import host_popcount_peak
    cores = os.cpu_count()
    res = {"host": host_popcount_peak(cores), "cores": cores, "runs": []}

    def rec(name, mode, threads, r, full_cmp):
        rate = r["cmp"] / r["seconds"]
        res["runs"].append({"config": name, "mode": mode, "threads": threads, "seconds": round(r["seconds"], 3),
                            "comparisons": r["cmp"], "cmp_per_s": rate,
                            "full_workload_seconds": round(full_cmp / rate, 1)})
        print(json.dumps(res["runs"][-1]), file=sys.stderr, flush=True)

    # configs[0] LD-2K: full, all cores and one thread
    full = 2048 * 2048 * 4096
    rec("ld2k", "full", cores, run("ld", 1001, 2048, 2048, 4096), full)
    rec("ld2k", "full", 1, run("ld", 1001, 2048, 2048, 4096, threads=1), full)
    # configs[1] FastID-1M: full (64 queries x 1M rows x 4096 SNPs, XOR + ANDNOT)
    full = 2 * 64 * 1_000_000 * 4096
    rec("fastid1m", "full", cores, run("fastid", 1002, 1_000_000, 1_000_000, 4096, 64), full)
    # configs[2] LD-32K: 256 seeded rows against all 32,768 columns, extrapolated
    full = 32768 * 32768 * 16384
    rec("ld32k", "extrapolated (256 rows x 32768 SNPs)", cores, run("ld", 1003, 256, 32768, 16384), full)
    # configs[3] FastID-20M: 1,024 queries x 20,000 rows, extrapolated to 20M rows
    full = 2 * 1024 * 20_000_000 * 8192
    rec("fastid20m", "extrapolated (1024 queries x 20000 rows)", cores,
        run("fastid", 1004, 20_000, 20_000_000, 8192, 1024), full)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    t0 = time.time()
    main()
    print(f"total {time.time() - t0:.0f} s", file=sys.stderr)
