"""Per-operator profile of the 13 SSB plans (event-timed replay + byte model).

usage: python tools/opprofile.py [--sf 20] [--queries ssb1.1,ssb3.1] [--launch N] [--json OUT]
  --launch N: only launch each prepared plan N times (for ncu), no table.
  --json OUT: also write per-class launches / algorithmic bytes per launch / event
  time per launch (tools/ncu_traffic.py joins it with the ncu DRAM bytes).
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--queries", default="")
    ap.add_argument("--launch", type=int, default=0)
    ap.add_argument("--json", default="")
    ap.add_argument("--star", action="store_true", help="n-ary STAR operator instead of binary-operator chains")
    ap.add_argument("--world", type=int, default=1,
                    help="dimensions of SF sf*W, lineorder = rank 0's shard of W (a weak-scaling rank)")
    a = ap.parse_args()
    import torch
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan
    qs = a.queries.split(",") if a.queries else SSB_QUERIES
    data = datagen.SSB(a.sf * a.world)
    db = Database(cache_bytes=64 << 30, heap_bytes=24 << 30)
    if a.world > 1:
        e = data.rows("lineorder") // a.world
        sf_total = a.sf * a.world

        class Shard:  # dimensions whole, lineorder rows [0, e) only
            def __getitem__(self, col):
                return datagen.ssb_column(col, sf_total, begin=0, end=e) if col.startswith("lo_") else data[col]

            def rows(self, t):
                return data.rows(t)

            def dict_for(self, col):
                return data.dict_for(col)
        load_ssb(db, Shard(), row_begin=0, row_end=e, presliced=True)
    else:
        load_ssb(db, data)
    preps = {q: db.prepare(ssb_plan(db, q, star=a.star)) for q in qs}
    torch.cuda.synchronize()
    if a.launch:
        for _ in range(a.launch):
            for p in preps.values():
                p.launch()
        torch.cuda.synchronize()
        return
    names = {0: "dense", 1: "at-tids", 2: "build", 3: "gather", 4: "agg", 5: "masked"}
    tot = {}
    # whole-graph time per query (the plan's CUDA graph, branches overlapped)
    stream = torch.cuda.Stream()
    gsum = 0.0
    for q, p in preps.items():
        for _ in range(3):
            p.launch(stream.cuda_stream)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(20):
            p.launch(stream.cuda_stream)
        e1.record(stream)
        torch.cuda.synchronize()
        g = e0.elapsed_time(e1) / 20
        gsum += g
        print(f"{q} graph {g*1e3:.0f}us")
    print(f"graphs   {gsum*1e3:9.0f} us (sum of per-query graph times)")
    for q, p in preps.items():
        for _ in range(3):
            p.launch()
        prof = p.profile()
        prof = p.profile()
        ops = p.db  # noqa
        line = []
        for i, (ms, by, cl) in enumerate(prof):
            line.append(f"{names[cl]}:{ms*1e3:.0f}us/{by/1e6:.0f}MB/{by/ms/1e6 if ms else 0:.0f}GB/s")
            t = tot.setdefault(names[cl], [0.0, 0.0, 0])
            t[0] += ms
            t[1] += by
            t[2] += 1
        print(q, f"total {sum(x[0] for x in prof)*1e3:.0f}us", " | ".join(line))
    for k, (ms, by, n) in tot.items():
        print(f"{k:8s} {ms*1e3:9.0f} us {by/1e9:8.3f} GB {by/ms/1e6:8.0f} GB/s")
    if a.json:
        import json
        json.dump({"sf": a.sf, "queries": qs, "per_step": {
            k: {"launches": n, "algorithmic_bytes_per_launch": round(by / n), "event_us_per_launch": round(ms * 1e3 / n, 2)}
            for k, (ms, by, n) in tot.items()}}, open(a.json, "w"), indent=1)


if __name__ == "__main__":
    main()
