"""Kernel timeline of bench.py's hot step (CUPTI activity records via torch.profiler).

usage: python tools/timeline.py [--sf 20] [--streams 4] [--steps 3] --out gpurun_out/tl.json
Writes every kernel / memset of the traced steps: name, stream, start and duration
(us, relative to the first), and prints per-step wall time, the busy fraction of the
device (any kernel running) and the per-kernel-class sums, so the overlap of the
K query streams (and the latency-bound tails between big kernels) can be read off.
The timed bench number never comes from here (the tracer adds launch overhead).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--streams", type=int, default=4)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/timeline.json")
    a = ap.parse_args()
    import torch
    from torch.profiler import ProfilerActivity, profile
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan

    data = datagen.SSB(a.sf)
    db = Database(cache_bytes=64 << 30, heap_bytes=24 << 30)
    load_ssb(db, data)
    preps = [db.prepare(ssb_plan(db, q), use_graph=True) for q in SSB_QUERIES]
    main_s = torch.cuda.Stream()
    side = [torch.cuda.Stream() for _ in range(a.streams - 1)]
    lanes = [main_s] + side

    def step():
        for s in side:
            s.wait_stream(main_s)
        for i, p in enumerate(preps):
            p.launch(lanes[i % len(lanes)].cuda_stream)
        for s in side:
            main_s.wait_stream(s)

    for _ in range(5):
        step()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(a.steps):
            step()
        torch.cuda.synchronize()
    evs = []
    for e in prof.events():
        if e.device_type.name != "CUDA":
            continue
        evs.append({"name": e.name, "stream": getattr(e, "device_resource_id", -1),
                    "ts": e.time_range.start, "dur": e.time_range.end - e.time_range.start})
    evs.sort(key=lambda x: x["ts"])
    t0 = evs[0]["ts"] if evs else 0
    for x in evs:
        x["ts"] -= t0
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    json.dump({"sf": a.sf, "streams": a.streams, "steps": a.steps, "queries": SSB_QUERIES, "events": evs},
              open(a.out, "w"))
    # busy fraction: union of kernel intervals over the traced span
    iv = sorted((x["ts"], x["ts"] + x["dur"]) for x in evs)
    busy, cur_s, cur_e = 0.0, None, None
    for s, e in iv:
        if cur_e is None or s > cur_e:
            if cur_e is not None:
                busy += cur_e - cur_s
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    if cur_e is not None:
        busy += cur_e - cur_s
    span = max(e for _, e in iv) - min(s for s, _ in iv) if iv else 0
    tot = sum(x["dur"] for x in evs)
    print(f"events {len(evs)} span {span:.0f} us ({span / a.steps:.0f} us/step) busy {busy / max(span, 1):.3f} "
          f"sum-of-durations/span {tot / max(span, 1):.2f}")


if __name__ == "__main__":
    main()
