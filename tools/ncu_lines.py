"""Aggregate an ncu source page (cuda,sass) per CUDA source line.

usage: python tools/ncu_lines.py REPORT LAUNCH_INDEX [N]
Prints the N source lines with the most stall samples, their share of executed
instructions and top stall reasons.
"""
import csv
import io
import subprocess
import sys


def f(x):
    try:
        return float(x.replace(",", ""))
    except ValueError:
        return 0.0


def main():
    rep, skip = sys.argv[1], sys.argv[2]
    n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass", "--launch-skip",
                          skip, "--launch-count", "1"], capture_output=True, text=True).stdout
    fname, cur, h = "?", None, None
    agg = {}
    for r in csv.reader(io.StringIO(out)):
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            h = r
            continue
        if h is None or len(r) != len(h):
            continue
        if r[0]:
            cur = (fname, int(r[0]), r[1].strip())
            continue
        d = dict(zip(h[2:], r[2:]))
        a = agg.setdefault(cur, {"s": 0.0, "i": 0.0, "st": {}})
        a["s"] += f(d["# Samples"])
        a["i"] += f(d["Instructions Executed"])
        for c in h[2:]:
            if c.startswith("stall_") and "Not Issued" not in c:
                a["st"][c[6:]] = a["st"].get(c[6:], 0.0) + f(d[c])
    ts = sum(a["s"] for a in agg.values()) or 1
    ti = sum(a["i"] for a in agg.values()) or 1
    print(f"samples {ts:.0f}  warp-instructions {ti:.0f}")
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["s"])[:n]:
        st = sorted(((v, c) for c, v in a["st"].items()), reverse=True)[:3]
        name = f"{k[0]}:{k[1]}" if k else "?"
        src = k[2][:70] if k else ""
        print(f"{name:24s} {100*a['s']/ts:5.1f}% samp {100*a['i']/ti:5.1f}% inst | {src:70s} | "
              + " ".join(f"{c}:{100*v/max(a['s'],1):.0f}%" for v, c in st))


if __name__ == "__main__":
    main()
