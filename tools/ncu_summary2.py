"""Summarise an ncu --set full report: per kernel launch, time, DRAM bytes, L1
wavefronts, issue activity and the top stall reasons.
usage: python tools/ncu_summary2.py report.ncu-rep"""
import csv
import subprocess
import sys

KEYS = [("gpu__time_duration.sum", "us", 1e-3), ("dram__bytes_read.sum", "MB_rd", 1e-6),
        ("dram__bytes_write.sum", "MB_wr", 1e-6), ("smsp__inst_executed.sum", "Minst", 1e-6),
        ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue%", 1),
        ("l1tex__throughput.avg.pct_of_peak_sustained_active", "l1%", 1),
        ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2%", 1),
        ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram%", 1),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "occ%", 1),
        ("launch__registers_per_thread", "regs", 1), ("launch__grid_size", "grid", 1),
        ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "Mwf_smem", 1e-6),
        ("l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_ld.sum", "Mwf_gld", 1e-6)]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    idx = {k: h.index(k) for k, _, _ in KEYS if k in h}
    name_i = h.index("Kernel Name")
    for r in rows[2:]:
        parts = []
        for k, lab, sc in KEYS:
            if k in idx:
                try:
                    unit = rows[1][idx[k]]
                    v = float(r[idx[k]].replace(",", ""))
                    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "byte": 1e-6, "Kbyte": 1e-3,
                             "Mbyte": 1.0, "Gbyte": 1e3}.get(unit)
                    if lab in ("us", "MB_rd", "MB_wr") and scale is not None:
                        v = v * scale
                    else:
                        v = v * sc
                    parts.append(f"{lab}={v:.1f}")
                except ValueError:
                    pass
        stalls = []
        for i, x in enumerate(h):
            if x.startswith("smsp__average_warps_issue_stalled_") and x.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(r[i]), x[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        print(r[name_i][:70])
        print("   " + " ".join(parts))
        print("   stalls: " + ", ".join(f"{n} {v:.2f}" for v, n in stalls[:6]))


if __name__ == "__main__":
    main(sys.argv[1])
