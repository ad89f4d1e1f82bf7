"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck): every
kernel family of libddq at tiny sizes -- all 13 SSB queries (STAR, chain, eager,
fused-tail and unfused plans; dense and sparse keys, i.e. join indexes and hash
tables), TPC-H Q1-Q7 (dense aggregation, MIN, key sets, FILTER_EQ), prepared plans
WITHOUT graphs (each kernel launched directly) and through the chopping driver --
each result checked against the oracle.

usage: compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import datagen
    import oracle
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan
    from paper_conf_sigmod_bressft16_b200.tpch import TPCH_QUERIES, load_tpch, tpch_plan
    n = 0
    for keys in ("dense", "sparse"):
        data = datagen.SSB(0.02, keys=keys)
        db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30)
        load_ssb(db, data)
        for q in SSB_QUERIES:
            want = oracle.run(data, q)
            for kw in (dict(), dict(star=True), dict(late=False), dict(fuse_tail=True),
                       dict(fused_build=False, late=False, fused_agg=False)):
                p = db.prepare(ssb_plan(db, q, **kw), use_graph=False)
                p.launch()
                assert p.fetch().rows == want, (keys, q, kw)
                p.close()
                n += 1
            assert db.run(ssb_plan(db, q)).rows == want, (keys, q)
        db.close()
        td = datagen.TPCH(0.02, keys=keys)
        db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30)
        load_tpch(db, td)
        for q in TPCH_QUERIES:
            want = oracle.run(td, q)
            p = db.prepare(tpch_plan(db, q), use_graph=False)
            p.launch()
            assert p.fetch().rows == want, (keys, q)
            p.close()
            assert db.run(tpch_plan(db, q)).rows == want, (keys, q)
            n += 1
        db.close()
    print(f"sanitize_run: {n} plans equal the oracle")


if __name__ == "__main__":
    main()
