"""M1 (BASELINE configs[0]): SSB Q1.1 at SF1 (6 M lineorder rows), one
query, hot cache, 1 GPU, the paper's protocol -- 2 warm-up runs then 100 timed runs
 -- with L2 flushed before every run (a write of 2x the L2 size), timed with
CUDA events on the launch stream; the prepared plan launched as one CUDA graph and
as plain kernel launches (use_graph=False).  Prints one JSON line.

usage: python tools/m1.py [--runs 100] [--out profiles/r2_m1.json]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--runs", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    import datagen
    import oracle
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import load_ssb, ssb_plan

    torch.cuda.set_device(0)
    data = datagen.SSB(1)
    db = Database(cache_bytes=8 << 30, heap_bytes=4 << 30)
    load_ssb(db, data)
    want = oracle.run(data, "ssb1.1")
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    scrub = torch.empty(2 * l2 // 4, dtype=torch.int32, device="cuda")
    stream = torch.cuda.Stream()
    res = {}
    for mode in ("graph", "plain"):
        p = db.prepare(ssb_plan(db, "ssb1.1"), use_graph=(mode == "graph"))
        times = []
        for i in range(a.warmup + a.runs):
            with torch.cuda.stream(stream):
                scrub.fill_(i)  # evict the previous run's lines from L2
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            p.launch(stream.cuda_stream)
            e1.record(stream)
            e1.synchronize()
            if i >= a.warmup:
                times.append(e0.elapsed_time(e1) * 1e3)
        got = p.fetch(stream.cuda_stream).rows
        assert got == want, (got, want)
        p.close()
        med = statistics.median(times)
        res[mode] = {"us_median": round(med, 2), "us_min": round(min(times), 2), "us_max": round(max(times), 2),
                     "rows_per_s": 6_000_000 / (med / 1e6), "kernels": None}
    line = {"config": "M1: SSB Q1.1, SF1 (6 M lineorder rows), hot cache, 1 GPU, L2 flushed before each run",
            "protocol": f"{a.warmup} warm-ups + {a.runs} timed runs (P:305), CUDA events, median",
            "result_equals_oracle": True, **res,
            "gpu": torch.cuda.get_device_name(0)}
    print(json.dumps(line))
    if a.out:
        with open(a.out, "w") as f:
            f.write(json.dumps(line, indent=1) + "\n")
    db.close()


if __name__ == "__main__":
    main()
