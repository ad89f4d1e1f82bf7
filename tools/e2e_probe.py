"""Diagnose the cold-cache end-to-end path (bench.py e2e): per-query wall time and
driver statistics with GPU-only placement on an empty cache."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan
    sf = float(sys.argv[1]) if len(sys.argv) > 1 else 20
    data = datagen.SSB(sf)
    cold = Database(cache_bytes=64 << 30, heap_bytes=24 << 30, placement=A.PLACE_GPU_ONLY)
    t0 = time.perf_counter()
    load_ssb(cold, data, cache=False)
    print(f"load {time.perf_counter() - t0:.2f}s", flush=True)
    plans = [ssb_plan(cold, q) for q in SSB_QUERIES]
    for rep in range(2):
        cold.reset_stats()
        tq = time.perf_counter()
        for q, pl in zip(SSB_QUERIES, plans):
            t = time.perf_counter()
            cold.run(pl)
            st = cold.stats()
            print(f"  {q} {1e3 * (time.perf_counter() - t):8.1f} ms  h2d {st['h2d_bytes'] / 1e9:6.2f} GB "
                  f"{st['h2d_ns'] / 1e6:8.1f} ms  host_ops {st['host_ops']} aborts {st['aborts']}", flush=True)
        t = time.perf_counter()
        for (tb, c) in list(cold._cols):
            cold.evict(tb, c)
        print(f"rep {rep}: queries {1e3 * (t - tq):.1f} ms, evict {1e3 * (time.perf_counter() - t):.1f} ms", flush=True)
        # concurrent submission
        cold.reset_stats()
        t = time.perf_counter()
        qs = [cold.submit(pl) for pl in plans]
        for h in qs:
            cold.fetch(h)
        st = cold.stats()
        print(f"rep {rep}: concurrent {1e3 * (time.perf_counter() - t):.1f} ms h2d {st['h2d_bytes'] / 1e9:.2f} GB "
              f"{st['h2d_ns'] / 1e6:.1f} ms", flush=True)
        for (tb, c) in list(cold._cols):
            cold.evict(tb, c)
    cold.close()


if __name__ == "__main__":
    main()
