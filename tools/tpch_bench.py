"""BASELINE config 4: TPC-H Q1/Q3/Q5/Q6 at SF30 (plus Q4/Q7, S8(f) N2), hot and cold cache.

hot : prepared plans (CUDA graphs) over resident columns, CUDA-event timed,
      lineitem rows/s per query;
cold: GPU-only placement on an empty cache through ddq_submit/ddq_fetch: every
      column is copied from pinned host memory inside the timed region (the
      paper's cold case); reports H2D GB/s against the link.
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=30)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--ops", action="store_true", help="also print the per-operator profile (stderr)")
    a = ap.parse_args()
    import torch
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.tpch import TPCH_QUERIES, load_tpch, tpch_plan
    data = datagen.TPCH(a.sf)
    n = data.rows("lineitem")
    db = Database(cache_bytes=100 << 30, heap_bytes=40 << 30)
    load_tpch(db, data)
    st = torch.cuda.Stream()
    for q in TPCH_QUERIES:
        p = db.prepare(tpch_plan(db, q, limit=10 if q == "tpch3" else 0), use_graph=True)
        for _ in range(3):
            p.launch(st.cuda_stream)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(a.steps):
            p.launch(st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.steps
        rows = p.fetch(st.cuda_stream).rows
        prof = p.profile(st.cuda_stream)
        byt = sum(b for _, b, _ in prof)
        if a.ops:
            names = {0: "dense", 1: "at-tids", 2: "build", 3: "gather", 4: "agg", 5: "masked"}
            print(q, " | ".join(f"{names.get(c, c)}:{m * 1e3:.0f}us/{b / 1e6:.0f}MB" for m, b, c in prof),
                  file=sys.stderr, flush=True)
        print(json.dumps({"config": "M4", "mode": "hot", "query": q, "sf": a.sf, "lineitem_rows": n,
                          "ms": round(ms, 4), "rows_per_s": n / (ms / 1e3), "model_gb": round(byt / 1e9, 3),
                          "model_gbs": round(byt / (ms / 1e3) / 1e9, 1), "groups": len(rows)}), flush=True)
        p.close()
    db.close()
    for mode in ("cold", "cold_streamed"):
        cold_run(A, Database, load_tpch, tpch_plan, TPCH_QUERIES, data, a, n, mode)


def cold_run(A, Database, load_tpch, tpch_plan, TPCH_QUERIES, data, a, n, mode):
    """cold: columns copied when an operator needs them; cold_streamed: the streamed
    cold path (ddq_config.prefetch, S8(f) N1): the plan's columns stream in from submit
    while earlier operators compute."""
    cold = Database(cache_bytes=100 << 30, heap_bytes=40 << 30, placement=A.PLACE_GPU_ONLY,
                    prefetch=(mode == "cold_streamed"))
    load_tpch(cold, data, cache=False)
    cols = list(cold._cols)
    for q in TPCH_QUERIES:
        plan = tpch_plan(cold, q, limit=10 if q == "tpch3" else 0)
        cold.run(plan)
        for (t, c) in cols:
            cold.evict(t, c)
        cold.reset_stats()
        t0 = time.perf_counter()
        r = cold.run(plan)
        dt = time.perf_counter() - t0
        s = cold.stats()
        for (t, c) in cols:
            cold.evict(t, c)
        print(json.dumps({"config": "M4", "mode": mode, "query": q, "sf": a.sf, "ms": round(dt * 1e3, 2),
                          "rows_per_s": n / dt, "h2d_bytes": s["h2d_bytes"],
                          "h2d_gbs": round(s["h2d_bytes"] / max(s["h2d_ns"], 1), 2),
                          "h2d_gbs_wall": round(s["h2d_bytes"] / dt / 1e9, 2), "groups": len(r.rows),
                          "host_ops": r.host_ops}), flush=True)
    cold.close()


if __name__ == "__main__":
    main()
