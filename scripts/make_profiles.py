"""Summarise gpurun_out/prof/* (ncu launch lists + --set full captures) into profiles/<round>/.

Writes human-readable summaries and profiles/traffic.json (dram read+write bytes per
launch of the dominant kernel, keyed "<workload>:<kernel>") that bench.py reports as
roofline.traffic."""
import csv, json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "gpurun_out", "prof")
ROUND = sys.argv[1] if len(sys.argv) > 1 else "round1"
DST = os.path.join(ROOT, "profiles", ROUND)
os.makedirs(DST, exist_ok=True)

def short(name):
    for key in ("gemm_tc4x2_kernel", "fastid_tc4_kernel", "fastid_stream_kernel", "gemm_tc4_kernel", "bitgemm_popc_kernel", "bitgemm_tc_kernel",
                "pack_popc_kernel", "pack_vec_kernel", "pack_byte_kernel", "row_popc_kernel", "sym_unpack_kernel",
                "fastid_search_init", "stream_search_init", "best_init", "best_reduce", "best_finalize"):
        if key in name:
            return key
    return name.split("(")[0][-60:]

def launches(path, per_step, steps_keep):
    rows = [r for r in csv.reader(l for l in open(path) if not l.startswith("=="))]
    hdr = rows[0]
    ik, iv, im = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
    ks = [(short(r[ik]), float(r[iv])) for r in rows[1:] if r[im] == "gpu__time_duration.sum"]
    ks = ks[-per_step * steps_keep:]
    tot = sum(v for _, v in ks)
    agg = {}
    for k, v in ks:
        agg.setdefault(k, [0, 0.0])
        agg[k][0] += 1
        agg[k][1] += v
    return ks, tot, agg

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return [{h: (v, u) for h, v, u in zip(rows[0], r, rows[1])} for r in rows[2:]]

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "smsp__warps_active.avg.per_cycle_active"]

def to_bytes(v, u):
    f = float(v)
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)

traffic = {}
tpath = os.path.join(ROOT, "profiles", "traffic.json")
if os.path.exists(tpath):
    traffic = json.load(open(tpath))
summary = []
for wl, per_step in (("fastid1m", 3), ("ld32k", 2), ("ld2k", 2), ("fastid20m", 7)):
    p = os.path.join(SRC, f"launches_{wl}.csv")
    if os.path.exists(p):
        ks, tot, agg = launches(p, per_step, 2)
        summary.append(f"## launch list {wl} (ncu gpu__time_duration.sum, cold-cache serialised; last 2 steps, {len(ks)} launches)")
        for k, (n, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
            summary.append(f"  {k:24s} launches {n:3d}  total {v / 1e3:10.1f} us  share {100 * v / tot:5.1f} %")
for name, wl, kern in (("full_fastid1m", "fastid1m", "fastid_mxf4"), ("full_ld32k", "ld32k", "tc_mxf4_sym_pair"),
                       ("full_ld2k", "ld2k", "tc_mxf4_sym"), ("full_fastid20m", "fastid20m", "tc_mxf4"),
                       ("full_fastid1m_popc", "fastid1m", "popc"), ("full_stream1", "skinny1x20Mx4096", "popc_stream"),
                       ("full_skinny8", "skinny8x20Mx4096", "fastid_mxf4")):
    rep = os.path.join(SRC, name + ".ncu-rep")
    if not os.path.exists(rep):
        continue
    for d in raw(rep):
        kname = short(d.get("Kernel Name", ("?",))[0])
        summary.append(f"## ncu --set full: {name} ({kname})")
        for k in KEYS:
            if k in d:
                summary.append(f"  {k} = {d[k][0]} {d[k][1]}")
        st = [(k, v) for k, v in d.items() if k.startswith("smsp__average_warps_issue_stalled") and k.endswith("per_issue_active.ratio")]
        st.sort(key=lambda x: -float(x[1][0] or 0))
        summary.append("  top stalls/issue: " + ", ".join(
            f"{k.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')}={float(v[0]):.2f}" for k, v in st[:6]))
        rb = to_bytes(*d["dram__bytes_read.sum"]) if "dram__bytes_read.sum" in d else None
        wb = to_bytes(*d["dram__bytes_write.sum"]) if "dram__bytes_write.sum" in d else None
        if rb is not None and wb is not None:
            traffic[f"{wl}:{kern}"] = rb + wb
            summary.append(f"  dram traffic per launch = {(rb + wb) / 1e6:.1f} MB")
open(os.path.join(DST, "summary.txt"), "w").write("\n".join(summary) + "\n")
json.dump(traffic, open(tpath, "w"), indent=1)
print("\n".join(summary))
