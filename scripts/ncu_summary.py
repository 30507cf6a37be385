"""Summarise an ncu --set full report (raw page) into the key roofline/stall numbers."""
import csv, subprocess, sys
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
hdr, units = rows[0], rows[1]
for vals in rows[2:]:
    d = {h: (v, u) for h, v, u in zip(hdr, vals, units)}
    print("kernel:", d.get("Kernel Name", ("?",))[0][:90])
    keys = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
            "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
            "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
            "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "lts__t_bytes.sum.per_second", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "launch__registers_per_thread", "smsp__warps_active.avg.per_cycle_active"]
    for k in keys:
        if k in d:
            print(f"  {k} = {d[k][0]} {d[k][1]}")
    st = [(k, v) for k, v in d.items() if k.startswith("smsp__average_warps_issue_stalled") and k.endswith("per_issue_active.ratio")]
    st.sort(key=lambda x: -float(x[1][0] or 0))
    print("  stalls/issue:", ", ".join(f"{k.replace('smsp__average_warps_issue_stalled_','').replace('_per_issue_active.ratio','')}={float(v[0]):.2f}" for k, v in st[:7]))
