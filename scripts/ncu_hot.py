"""Print the hottest SASS lines (warp stall samples) of an ncu report with their stall reasons."""
import csv, subprocess, sys
rep = sys.argv[1]; n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]; data = rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
ri = [hdr.index(r) for r in reasons]
tot = sum(int(r[i_s] or 0) for r in data)
print("total samples", tot)
top = sorted(range(len(data)), key=lambda k: -int(data[k][i_s] or 0))[:n]
for k in sorted(top):
    r = data[k]
    rs = sorted(((int(r[i] or 0), reasons[j][6:]) for j, i in enumerate(ri)), reverse=True)[:2]
    print(f"{k:5d} {r[i_s]:>5} {r[1][:70]:70s} {rs}")
