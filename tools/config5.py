"""BASELINE config 5 / SURVEY 8(d) M5: concurrent SSB streams whose working set
exceeds the device budget -- data-driven query chopping vs naive GPU placement vs
CPU only (the paper's Sec. 6.2.2 experiment, Fig. 18-20).

Fixed total work: `--queries` queries = seeded permutations of the 13,
split round-robin over U user threads that submit through the C ABI
(ddq_submit/ddq_fetch; ctypes releases the GIL).  Device budget: a column cache of
`--cache-frac` of the 13-query working set and a small heap.

Arms (Sec. 6.2)
  ddc        data-driven placement + chopping; Algorithm 1 (LFU) fills the cache
             from the access counts of one warm-up pass
  chopping   run-time placement with the bounded pull queues on the
             GPU-only arm: columns copied on demand (LRU), gpu_workers operators at once
  gpu_only   operator-driven placement at compile time, columns copied on demand
             with LRU eviction, no concurrency bound ("GPU Preferred")
  admission  gpu_only with query-level admission control: one query at a time
             (ddq_config.max_queries = 1; Wang et al., the reference point of P:371)
  cpu_only   host executor only
Prints one JSON line per (arm, users): makespan, queries/s, H2D bytes/time,
aborts, wasted time, latency p50/p95, and checks every result against the first
arm's (placement never changes results).
"""
import argparse
import json
import os
import random
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--users", default="1,8,16,32")
    ap.add_argument("--queries", type=int, default=104)
    ap.add_argument("--cache-frac", type=float, default=0.5)
    ap.add_argument("--heap-gb", type=float, default=1.0)
    ap.add_argument("--arms", default="ddc,chopping,gpu_only,admission,cpu_only")
    ap.add_argument("--policy", default="lfu", choices=["lfu", "lru"], help="Algorithm 1 ordering (App. E)")
    ap.add_argument("--host-workers", type=int, default=4)
    ap.add_argument("--gpu-workers", type=int, default=4)
    a = ap.parse_args()
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan, FACT_COLUMNS

    data = datagen.SSB(a.sf)
    n = data.rows("lineorder")
    ws_bytes = sum(data[c].nbytes for c in FACT_COLUMNS)
    cache_bytes = int(a.cache_frac * ws_bytes)
    rng = random.Random(2016)
    work = []
    while len(work) < a.queries:
        p = list(SSB_QUERIES)
        rng.shuffle(p)
        work += p
    work = work[:a.queries]
    reference = {}
    for arm in a.arms.split(","):
        for U in [int(u) for u in a.users.split(",")]:
            kw = dict(cache_bytes=cache_bytes, heap_bytes=int(a.heap_gb * (1 << 30)), gpu_workers=a.gpu_workers,
                      host_workers=a.host_workers, cache_policy=1 if a.policy == "lru" else 0)
            if arm == "ddc":
                kw.update(placement=A.PLACE_DATA_DRIVEN, chopping=True)
            elif arm == "chopping":
                kw.update(placement=A.PLACE_GPU_ONLY, chopping=True)
            elif arm == "gpu_only":
                kw.update(placement=A.PLACE_GPU_ONLY, chopping=False)
            elif arm == "admission":
                kw.update(placement=A.PLACE_GPU_ONLY, chopping=False, max_queries=1)
            else:
                kw.update(placement=A.PLACE_CPU_ONLY, chopping=True)
            db = Database(**kw)
            load_ssb(db, data, cache=False)
            plans = {q: ssb_plan(db, q) for q in SSB_QUERIES}
            if arm == "ddc":  # one warm-up pass to learn access counts, then Algorithm 1
                for q in SSB_QUERIES:
                    db.run(plans[q])
                db.update_placement()
            db.reset_stats()
            lat = []
            results = {}
            lock = threading.Lock()

            def user(u):
                for i in range(u, len(work), U):
                    q = work[i]
                    t0 = time.perf_counter()
                    r = db.run(plans[q])
                    dt = time.perf_counter() - t0
                    with lock:
                        lat.append(dt)
                        results.setdefault(q, r.rows)
            t0 = time.perf_counter()
            th = [threading.Thread(target=user, args=(u,)) for u in range(U)]
            for t in th:
                t.start()
            for t in th:
                t.join()
            makespan = time.perf_counter() - t0
            st = db.stats()
            lat.sort()
            for q, rows in results.items():
                if q in reference:
                    assert rows == reference[q], (arm, U, q)
                else:
                    reference[q] = rows
            line = {"config": "M5", "arm": arm, "users": U, "sf": a.sf, "queries": len(work), "policy": a.policy,
                    "cache_bytes": cache_bytes, "working_set_bytes": ws_bytes, "heap_bytes": kw["heap_bytes"],
                    "makespan_s": round(makespan, 4), "queries_per_s": round(len(work) / makespan, 2),
                    "fact_rows_per_s": len(work) * n / makespan,
                    "h2d_bytes": st["h2d_bytes"], "h2d_s": st["h2d_ns"] / 1e9, "d2h_bytes": st["d2h_bytes"],
                    "gpu_ops": st["gpu_ops"], "host_ops": st["host_ops"], "aborts": st["aborts"],
                    "wasted_s": st["wasted_ns"] / 1e9, "heap_peak_bytes": st["heap_peak_bytes"],
                    "latency_p50_s": round(lat[len(lat) // 2], 4), "latency_p95_s": round(lat[int(len(lat) * .95)], 4),
                    "cached_columns": sum(1 for t, c in db._cols if db.is_cached(t, c)),
                    "results_equal": True}
            print(json.dumps(line), flush=True)
            db.close()


if __name__ == "__main__":
    main()
