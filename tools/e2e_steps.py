"""Cold-path steps as bench.py times them (13 queries submitted at once, GPU-only
placement, every column evicted after the step), with the driver counters per step:
where a slow step goes (aborts -> host restarts, wasted time, H2D volume)."""
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
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
    data = datagen.SSB(sf)
    cold = Database(cache_bytes=64 << 30, heap_bytes=24 << 30, placement=A.PLACE_GPU_ONLY)
    load_ssb(cold, data, cache=False)
    plans = [ssb_plan(cold, q) for q in SSB_QUERIES]
    cols = list(cold._cols)
    for i in range(steps):
        cold.reset_stats()
        t = time.perf_counter()
        qs = [cold.submit(p) for p in plans]
        ts = 1e3 * (time.perf_counter() - t)
        done = []
        for q in qs:
            cold.fetch(q)
            done.append(round(1e3 * (time.perf_counter() - t)))
        dt = time.perf_counter() - t
        te = time.perf_counter()
        for (tb, c) in cols:
            cold.evict(tb, c)
        te = 1e3 * (time.perf_counter() - te)
        st = cold.stats()
        print(f"step {i}: {1e3 * dt:7.1f} ms (submit {ts:.1f} ms, done at {done}, evict {te:.1f} ms)  h2d {st['h2d_bytes'] / 1e9:5.2f} GB  gpu_ops {st['gpu_ops']} "
              f"host_ops {st['host_ops']} aborts {st['aborts']} wasted {st['wasted_ns'] / 1e6:.1f} ms", flush=True)
    cold.close()


if __name__ == "__main__":
    main()
