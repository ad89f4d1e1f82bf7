"""Per-kernel-class DRAM traffic and device time from an ncu launch list of the bench
command (ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
--csv --log-file X python bench.py --profile-only).

usage: python tools/ncu_traffic.py LAUNCHES.csv [OUT.json [MODEL.json]]
MODEL.json (tools/opprofile.py --json): the S8(d) algorithmic bytes per launch of each
class; with it every class also gets algorithmic_bytes_per_launch and
dram_over_algorithmic (> 1: bytes the model does not count -- 64-byte DRAM granules of
random gathers, L2 write-backs; < 1: reuse through L2).
Writes {class: {"launches", "dram_bytes_per_launch", "us_per_launch", "share"}}; bench.py
reads profiles/r2z_traffic.json to fill roofline.traffic for its dominant class.
Classes follow bench.py / ddq_prepared_profile: dense (ws_kernel, every row),
masked (ws_kernel over every row masked by a row bitmap), at-tids (ws_kernel over a
TID list, fetch_kernel), agg, build, other.
"""
import csv
import json
import re
import sys


def klass(name: str) -> str:
    m = re.search(r"ws_kernel<\s*(?:\(int\))?\s*\d+,\s*(?:\(int\))?\s*(\d+)", name)
    if m:
        return {"0": "dense", "2": "masked"}.get(m.group(1), "at-tids")
    if "scan_kernel" in name or "star_kernel" in name or "filter_kernel" in name:
        return "dense" if re.search(r"scan_kernel<\d+, (?:\(bool\))?(?:0|false)", name) else "at-tids"
    if "fetch_kernel" in name:  # late payload fetch through a join index: an at-TIDs lookup
        return "at-tids"
    if "agg_ws" in name or "agg_dense" in name or "groupby" in name:
        return "agg"
    if "build" in name:
        return "build"
    if "unpack" in name:  # load-time widening of packed columns (setup, not the step)
        return "load"
    return "other"


def main(path: str, out: str | None, model: str | None = None):
    rows = list(csv.reader(open(path)))
    h = None
    per = {}
    for r in rows:
        if r and r[0] == "ID":
            h = r
            continue
        if not h or len(r) != len(h):
            continue
        d = dict(zip(h, r))
        k = (d["ID"], d["Kernel Name"])
        v = float(d["Metric Value"].replace(",", ""))
        unit = d.get("Metric Unit", "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "ns": 1e-3,
                 "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1.0)
        per.setdefault(k, {})[d["Metric Name"]] = v * scale
    cls = {}
    for (i, name), m in per.items():
        c = klass(name)
        x = cls.setdefault(c, {"launches": 0, "bytes": 0.0, "us": 0.0})
        x["launches"] += 1
        x["bytes"] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        x["us"] += m.get("gpu__time_duration.sum", 0)
    tot = sum(x["us"] for x in cls.values()) or 1.0
    res = {c: {"launches": x["launches"], "dram_bytes_per_launch": round(x["bytes"] / x["launches"]),
               "us_per_launch": round(x["us"] / x["launches"], 2), "share": round(x["us"] / tot, 3)}
           for c, x in sorted(cls.items(), key=lambda t: -t[1]["us"])}
    if model:
        mc = json.load(open(model))["per_step"]
        for c, x in res.items():
            if c in mc:
                alg = mc[c]["algorithmic_bytes_per_launch"]
                x["algorithmic_bytes_per_launch"] = alg
                x["dram_over_algorithmic"] = round(x["dram_bytes_per_launch"] / alg, 3) if alg else None
    print(json.dumps(res, indent=1))
    if out:
        json.dump({"source": path, "model": model, "classes": res}, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, sys.argv[3] if len(sys.argv) > 3 else None)
