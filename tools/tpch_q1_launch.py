"""Launch TPC-H Q1's prepared plan N times (for ncu / timing of agg_dense_small_kernel).
usage: python tools/tpch_q1_launch.py [--sf 10] [--launch 2] [--time]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--launch", type=int, default=2)
    ap.add_argument("--time", action="store_true")
    ap.add_argument("--query", default="tpch1")
    a = ap.parse_args()
    import torch
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan
    data = datagen.TPCH(a.sf)
    db = Database(cache_bytes=60 << 30, heap_bytes=20 << 30)
    load_tpch(db, data)
    p = db.prepare(tpch_plan(db, a.query), use_graph=True)
    st = torch.cuda.Stream()
    for _ in range(a.launch):
        p.launch(st.cuda_stream)
    torch.cuda.synchronize()
    if a.time:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(20):
            p.launch(st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 20
        n = data.rows("lineitem")
        print(f"{a.query} sf{a.sf}: {ms:.3f} ms/query, {n * 44 / ms / 1e6:.0f} GB/s at 44 B/row")
    print(p.fetch(st.cuda_stream).rows[:2])


if __name__ == "__main__":
    main()
