"""Summarise tools/timeline.py output: per-kernel device time of one bench step (warm,
graph-launched) and, for a 1-stream trace, each query's kernel sequence.

usage: python tools/timeline_summary.py TIMELINE.json [TIMELINE.json ...]
"""
import json
import re
import sys
from collections import defaultdict


def short(name: str) -> str:
    m = re.search(r"(ws_kernel|agg_ws_kernel)<([^>]*)>", name)
    if m:
        args = m.group(2).replace("false", "0").replace("true", "1").replace(" ", "")
        return f"{m.group(1).replace('_kernel', '')}<{args}>"
    return re.sub(r"\(.*", "", name).replace("ddq::", "").replace("_kernel", "")[:24]


def main(paths):
    for path in paths:
        d = json.load(open(path))
        ev = d["events"]
        per = len(ev) // d["steps"]
        step = ev[:per]
        iv = sorted((x["ts"], x["ts"] + x["dur"]) for x in ev)
        span = iv[-1][1] - iv[0][0]
        print(f"== {path}: SF{d['sf']:g}, {d['streams']} stream(s), {d['steps']} traced steps, "
              f"{per} kernels/step, {span / d['steps']:.0f} us/step (under the tracer), "
              f"sum of kernel durations {sum(x['dur'] for x in ev) / span:.2f} x span")
        by = defaultdict(lambda: [0, 0.0, []])
        for e in step:
            k = short(e["name"])
            by[k][0] += 1
            by[k][1] += e["dur"]
            by[k][2].append(e["dur"])
        tot = sum(v[1] for v in by.values())
        print(f"  {'kernel':26s} {'n':>3s} {'us/step':>8s} {'share':>6s}  largest launches (us)")
        for k, (n, us, durs) in sorted(by.items(), key=lambda kv: -kv[1][1]):
            top = " ".join(f"{x:.0f}" for x in sorted(durs, reverse=True)[:8])
            print(f"  {k:26s} {n:3d} {us:8.1f} {us / tot:6.1%}  {top}")
        if d["streams"] == 1:  # one query after another: split at each plan's fill kernel
            print("  per query (kernel:us in graph order):")
            seqs, cur = [], []
            for e in step:
                k = short(e["name"])
                if k.startswith("multi_fill") and cur:
                    seqs.append(cur)
                    cur = []
                cur.append((k, e["dur"]))
            seqs.append(cur)
            for q, s in zip(d["queries"], seqs):
                print(f"  {q:7s} {sum(x for _, x in s):6.0f}  " + " ".join(f"{k}:{x:.0f}" for k, x in s))


if __name__ == "__main__":
    main(sys.argv[1:])
