"""Summarise an ncu report: per kernel duration, DRAM, occupancy, top stalls, top source lines."""
import csv, io, subprocess, sys
rep = sys.argv[1]
nlines = int(sys.argv[2]) if len(sys.argv) > 2 else 12
def run(args):
    return subprocess.run(["ncu", "-i", rep] + args, capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(run(["--page", "raw", "--csv"]))))
hdr, units = rows[0], rows[1]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "smsp__inst_executed.sum",
        "lts__t_bytes.sum", "l1tex__t_bytes.sum"]
for r in rows[2:]:
    v = dict(zip(hdr, r))
    print(f"ID {v['ID']} {v['Kernel Name'][:60]}")
    print("   " + "  ".join(f"{k.split('.')[0].replace('__','.')}={v.get(k)}{units[hdr.index(k)] if k in hdr else ''}" for k in keys if k in v))
    st = []
    for h, x in v.items():
        if "pcsamp_warps_issue_stalled" in h and not h.endswith("not_issued"):
            try:
                st.append((h.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(x.replace(",", ""))))
            except ValueError:
                pass
    st.sort(key=lambda t: -t[1])
    tot = sum(x for _, x in st) or 1
    print("   stalls: " + ", ".join(f"{h} {100*x/tot:.0f}%" for h, x in st[:7]))
