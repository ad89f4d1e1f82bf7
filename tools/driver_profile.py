"""Per-operator wall times of queries through the chopping driver (ddq_submit): the
result's op_ms (pull -> completion, incl. transfers and synchronisation) and the
query's exec_ms (submit -> root finished; finalisation is the rest of the fetch).

usage: python tools/driver_profile.py [--bench tpch|ssb] [--sf 30] [--queries tpch3] [--cold]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--bench", default="tpch")
    ap.add_argument("--sf", type=float, default=30)
    ap.add_argument("--queries", default="")
    ap.add_argument("--cold", action="store_true")
    a = ap.parse_args()
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    if a.bench == "tpch":
        from paper_conf_sigmod_bressft16_b200.tpch import TPCH_QUERIES as QS, load_tpch as load, tpch_plan as plan
        data = datagen.TPCH(a.sf)
    else:
        from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES as QS, load_ssb as load, ssb_plan as plan
        data = datagen.SSB(a.sf)
    qs = a.queries.split(",") if a.queries else QS
    kw = dict(placement=A.PLACE_GPU_ONLY, prefetch=True) if a.cold else {}
    db = Database(cache_bytes=100 << 30, heap_bytes=40 << 30, **kw)
    load(db, data, cache=not a.cold)
    cols = list(db._cols)
    for q in qs:
        p = plan(db, q, limit=10) if q == "tpch3" else plan(db, q)
        db.run(p)
        for _ in range(2):
            if a.cold:
                for (t, c) in cols:
                    db.evict(t, c)
            t0 = time.perf_counter()
            r = db.run(p)
            dt = time.perf_counter() - t0
        kinds = {1: "select", 2: "build", 3: "probe", 4: "gather", 5: "agg", 6: "filter", 7: "star"}
        ops = [f"{kinds.get(p.plan.ops[i].kind, '?')}:{m:.1f}" for i, m in enumerate(r.op_ms)]
        print(json.dumps({"query": q, "cold": a.cold, "wall_ms": round(dt * 1e3, 2), "exec_ms": round(r.exec_ms, 2),
                          "sum_op_ms": round(sum(r.op_ms), 2), "ops_ms": " ".join(ops)}), flush=True)
    db.close()


if __name__ == "__main__":
    main()
