"""Benchmark: all 13 SSB queries at SF20, hot cache, on B200 (BASELINE config 2,
the paper's Q3.3 setting); metric "SSB fact rows/s" (+ queries/s,
HBM GB/s vs peak).

One step = one pass of the whole hot path over the resident SF20 database: the 13
prepared physical plans (select -> build -> probe -> gather/aggregate, every
operator an sm_100a kernel of libddq) launched back to back on one stream.
value = 13 * lineorder_rows * steps / device time (CUDA events), max over ranks.
Inputs (6.7 GB of lineorder columns) are larger than L2 (126 MB), so no L2 flush
is needed between steps.

N > 1 (torchrun): lineorder is range-sharded by row (P:407 horizontal partitioning):
weak scaling by default (SF 20*N, 120 M rows per rank), strong scaling with
--sf-total 100 (S8(d) M3: 600 M rows split over the ranks).  libddq owns the
multi-GPU path (include/ddq.h "multi-GPU"): an NCCL communicator per database
(unique id bootstrapped through torch.distributed), per step one ncclAllGather of the
13 packed partial group tables, merged exactly by ddq_dist_result on rank 0; with
--build-once the dimension indexes are built on rank 0 and broadcast inside each
plan's CUDA graph (then one query stream: NCCL needs one collective order).

--impl reference: the oracle (oracle/, single-threaded C++) on a bounded sample
of the same workload, on the host's cores.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SSB fact rows/s"
UNIT = "rows/s"
SF_PER_GPU = 20.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--sf", type=float, default=SF_PER_GPU, help="scale factor per GPU (weak scaling)")
    ap.add_argument("--sf-total", type=float, default=0,
                    help="strong scaling (S8(d) M3): one database of this SF, lineorder row-sharded over the ranks")
    ap.add_argument("--build-once", action="store_true",
                    help="N>1: rank 0 builds the dimension indexes and NCCL broadcasts them inside the plan "
                         "graphs (one collective order: forces 1 query stream); default: every rank builds")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-prefetch", action="store_true", help="e2e: copy columns on demand instead of streaming")
    ap.add_argument("--dump-results", default="",
                    help="rank 0 writes the 13 (merged) query results of the timed plans as JSON (tests)")
    ap.add_argument("--emulate-world", type=int, default=0,
                    help="diagnostic: size the data for W ranks (dimensions of SF sf*W) and run rank 0's "
                         "lineorder shard on this single process (per-GPU step of a W-GPU weak-scaling run)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile-only", action="store_true", help="short run for ncu")
    ap.add_argument("--streams", type=int, default=0,
                    help="concurrent query streams inside a step: the 13 plans round-robin over K CUDA streams "
                         "(the paper's parallel users); 0 = pick the fastest of 1/2/4 from untimed trial steps")
    return ap.parse_args()


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class Clocks:
    """nvidia-smi clock / throttle sampling during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.p = None
        self.lines: list[str] = []

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None

    def _read(self):
        for line in self.p.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(2)
        except Exception:
            self.p.kill()
        self.t.join(1)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def host_facts() -> dict:
    """The host the CPU baseline runs on: online cores, CPU model, memory (S8(d))."""
    facts = {"nproc": os.cpu_count()}
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                facts["cpu"] = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal:"):
                facts["mem_gib"] = round(int(line.split()[1]) / (1 << 20), 1)
                break
    except OSError:
        pass
    return facts


class pinned_core:
    """Pin this process to one core (taskset -c 0 equivalent) while the
    single-threaded oracle is timed; the previous affinity is restored after."""

    def __init__(self, core: int = 0):
        self.core = core
        self.old = None

    def __enter__(self):
        try:
            self.old = os.sched_getaffinity(0)
            os.sched_setaffinity(0, {self.core if self.core in self.old else min(self.old)})
        except (AttributeError, OSError):
            self.old = None
        return self

    def __exit__(self, *exc):
        if self.old is not None:
            os.sched_setaffinity(0, self.old)


def cpu_baseline(sf: float, sample_rows: int, repeats: int = 3) -> dict:
    """The oracle as it stands (single-threaded C++), on the first `sample_rows`
    lineorder rows of the same SF database, all 13 queries; pinned to one core, the
    median of `repeats` runs (S8(d) oracle timing)."""
    import datagen
    import oracle
    data = datagen.SSB(sf)

    class Prefix:  # full dimension tables, lineorder prefix (generated only for the sample)
        def __getitem__(self, c):
            if c.startswith("lo_"):
                return datagen.ssb_column(c, sf, end=sample_rows)
            return data[c]
    pre = Prefix()
    cache = {}

    class View:
        def __getitem__(self, c):
            if c not in cache:
                cache[c] = pre[c]
            return cache[c]
    v = View()
    for q in oracle.SSB_QUERIES:  # generate inputs outside the timed region
        for c in oracle.SSB_QUERY_COLUMNS[int(q[3])]:
            v[c]
    runs = []
    with pinned_core(0):
        for _ in range(repeats):
            t0 = time.perf_counter()
            for q in oracle.SSB_QUERIES:
                oracle.run(v, q)
            runs.append(time.perf_counter() - t0)
    dt = sorted(runs)[len(runs) // 2]
    return {"value": 13 * sample_rows / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"all 13 SSB queries over the first {sample_rows} lineorder rows of SF{sf:g} "
                      f"(full dimension tables), single-threaded, pinned to core 0, median of {repeats} runs "
                      f"({', '.join(f'{x:.2f}' for x in runs)} s)",
            "host": host_facts()}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    import datagen  # noqa: F401
    sample = 2_000_000
    sf = args.sf * max(args.gpus, ws, 1)  # our arm's workload at N GPUs: SF 20 x N (weak scaling)
    vals = []
    for _ in range(args.warmup):
        cpu_baseline(sf, sample, repeats=1)
    t_total = 0.0
    for _ in range(args.steps):
        r = cpu_baseline(sf, sample, repeats=1)
        vals.append(r["value"])
        t_total += 13 * sample / r["value"]
    value = 13 * sample * args.steps / t_total
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_total / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64",
            "data": "synthetic (datagen, seed 0x5EED2016)",
            "config": {"workload": f"SSB SF{sf:g}, all 13 queries (bounded sample: first {sample} lineorder "
                                   f"rows per step)", "queries": 13},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"first {sample} lineorder rows of SF{sf:g} per step, pinned to core 0",
                             "host": host_facts()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import numpy as np
    import torch
    import datagen
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan, QUERY_COLUMNS
    QUERY_COLUMNS_ALL = sorted(set(sum(QUERY_COLUMNS.values(), [])))

    ws, rank, local = dist_env()
    assert ws == args.gpus or ws == 1, "launch N>1 with torchrun --nproc-per-node N"
    # DDQ_BENCH_BACKEND=gloo (test only): N ranks sharing the visible GPUs (rank ->
    # GPU local % count), to exercise the exchange and merge on a 1-GPU box
    backend = os.environ.get("DDQ_BENCH_BACKEND", "nccl")
    if backend != "nccl":
        local = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(local)
    if ws > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dws = args.emulate_world if (args.emulate_world and ws == 1) else ws  # ranks the data is sized for
    strong = args.sf_total > 0  # M3: one SF (e.g. 100) split over the ranks
    sf_total = args.sf_total if strong else args.sf * dws
    data = datagen.SSB(sf_total)
    n_lo = data.rows("lineorder")
    b, e = rank * n_lo // dws, (rank + 1) * n_lo // dws
    shard_rows = e - b

    class Shard:  # dimension tables whole, lineorder rows [b, e) only
        def __init__(self):
            self.c = {}

        def __getitem__(self, col):
            if col not in self.c:
                self.c[col] = (datagen.ssb_column(col, sf_total, begin=b, end=e) if col.startswith("lo_")
                               else data[col])
            return self.c[col]

        def rows(self, t):
            return data.rows(t)

        def dict_for(self, col):
            return data.dict_for(col)

    shard = Shard()
    t_setup = time.perf_counter()
    # heap: intermediates scale with the shard (24 GiB at SF20's 120 M rows)
    heap = min(110 << 30, max(24 << 30, int((24 << 30) * shard_rows / 120_000_000)))
    db = Database(device=local, cache_bytes=64 << 30, heap_bytes=heap, rank=rank, world=ws)
    if ws > 1:  # the library's multi-GPU exchange (S8(e)) before any plan is prepared
        import torch.distributed as dist
        if backend == "nccl":
            from paper_conf_sigmod_bressft16_b200.engine import nccl_unique_id
            box = [nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(box, src=0)
            db.dist_init_nccl(box[0], rank, ws, build_once=args.build_once)
        else:  # test hook: a host all-gather over the gloo process group
            def host_allgather(buf: bytes) -> bytes:
                t = torch.frombuffer(bytearray(buf), dtype=torch.uint8)
                out = [torch.empty_like(t) for _ in range(ws)]
                dist.all_gather(out, t)
                return b"".join(bytes(o.numpy()) for o in out)
            db.dist_init_host(rank, ws, host_allgather)

    load_ssb(db, shard, row_begin=b, row_end=e, presliced=True)
    if ws > 1:
        db.set_partitioned("lineorder")
    preps = [db.prepare(ssb_plan(db, q), use_graph=True) for q in SSB_QUERIES]
    setup_s = time.perf_counter() - t_setup
    stream = torch.cuda.Stream()
    sptr = stream.cuda_stream
    kernels_per_step = sum(p.kernels for p in preps)

    all_side = [torch.cuda.Stream() for _ in range(max(args.streams, 4) - 1)]
    side = all_side[:max(args.streams, 1) - 1]

    # the 13 plans are dealt round robin over the K streams in query order, which pairs
    # heavy and light plans on each stream (tried: longest-processing-time-first dealing
    # balanced the streams' solo times but started the four heaviest plans together and
    # measured slower, 2.66 -> 2.70 ms)
    def deal(k: int) -> list:
        return [i % k for i in range(len(preps))]
    lane_of = deal(1)

    def step(serial: bool = False):
        if serial or not side:
            for p in preps:
                p.launch(sptr)
            return
        lanes = [stream] + side
        for s2 in side:
            s2.wait_stream(stream)
        for i, p in enumerate(preps):
            p.launch(lanes[lane_of[i]].cuda_stream)
        for s2 in side:
            stream.wait_stream(s2)

    if args.streams == 0 and not args.profile_only:
        # untimed trial steps pick the stream count (4 at SF20; a dimension bitmap that
        # spills shared memory, e.g. customer at SF >= 60, makes concurrency lose)
        trial = {}
        for k in (1, 2, 4):
            side = all_side[:k - 1]
            lane_of = deal(k)
            step()
            ta, tb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            ta.record(stream)
            for _ in range(2):
                step()
            tb.record(stream)
            torch.cuda.synchronize()
            trial[k] = ta.elapsed_time(tb)
        if ws > 1:  # every rank uses the same count: the max-over-ranks time of each
            import torch.distributed as dist
            t = torch.tensor([trial[k] for k in (1, 2, 4)], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            trial = dict(zip((1, 2, 4), t.tolist()))
        args.streams = min(trial, key=trial.get)
    if args.build_once and ws > 1:  # NCCL broadcasts inside the graphs: one collective order
        args.streams = 1
    side = all_side[:max(args.streams, 1) - 1]
    lane_of = deal(max(args.streams, 1))

    # N>1: after the 13 launches, libddq packs the compacted partial group tables on the
    # device and all-gathers them (ncclAllGather over NVLink; the gloo test hook: a host
    # all-gather), and merges them exactly at finalisation (ddq_dist_exchange /
    # ddq_dist_result, S8(e)).
    def exchange():
        if ws > 1:
            db.dist_exchange(preps, sptr)

    def merged_results():
        """rank 0: every query's result over all ranks' rows."""
        return {q: db.dist_result(i).rows for i, q in enumerate(SSB_QUERIES)}

    if args.profile_only:
        for _ in range(2):
            step()
        torch.cuda.synchronize()
        return

    for _ in range(args.warmup):
        step()
        exchange()
    torch.cuda.synchronize()
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()
    clk = Clocks(local)
    clk.start()
    time.sleep(0.3)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    for _ in range(args.steps):
        step()
        exchange()
    ev1.record(stream)
    torch.cuda.synchronize()
    clocks = clk.stop()
    ms = ev0.elapsed_time(ev1)
    if ws > 1:
        import torch.distributed as dist
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        dist.barrier()
    ms_per_step = ms / args.steps
    fact_gb = sum(shard[c].nbytes for c in QUERY_COLUMNS_ALL) / 1e9
    l2_mb = torch.cuda.get_device_properties(local).L2_cache_size / 2**20
    total_rows = 13 * n_lo * ws // dws  # all ranks together (emulation: this shard only)
    value = total_rows * args.steps / (ms / 1e3)
    # the same K steps with the 13 plans back to back on one stream (per-query latency view)
    serial_ms = None
    if side:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(args.steps):
            step(serial=True)
            exchange()
        e1.record(stream)
        torch.cuda.synchronize()
        serial_ms = e0.elapsed_time(e1)
        if ws > 1:
            import torch.distributed as dist
            t = torch.tensor([serial_ms], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            serial_ms = float(t.item())

    # results of the timed plans (validated against the oracle by tests/, here sanity only)
    results = {q: p.fetch(sptr).rows for q, p in zip(SSB_QUERIES, preps)} if ws == 1 else \
        (merged_results() if rank == 0 else {})
    if args.dump_results and rank == 0:
        with open(args.dump_results, "w") as f:
            json.dump({q: [list(r) for r in rows] for q, rows in results.items()}, f)

    # ---- roofline of the dominant kernel class from an event-timed profiling replay
    prof = [p.profile(sptr) for p in preps]
    cls_ms, cls_bytes, cls_n = {}, {}, {}
    for ops in prof:
        for ms_, by, cl in ops:
            cls_ms[cl] = cls_ms.get(cl, 0.0) + ms_
            cls_bytes[cl] = cls_bytes.get(cl, 0.0) + by
            cls_n[cl] = cls_n.get(cl, 0) + 1
    names = {0: "ws_kernel (csrc/dense.cu): dense probe over all rows", 1: "ws_kernel (csrc/dense.cu): "
             "select/probe/fetch over a TID list", 2: "join_index_build_kernel (csrc/kernels.cu): build",
             3: "gather_kernel (csrc/kernels.cu)", 4: "agg_ws_kernel (csrc/agg.cu): group-by aggregate",
             5: "ws_kernel (csrc/dense.cu): probe of a key column masked by a row bitmap (every row streamed)"}
    tclass = {0: "dense", 1: "at-tids", 2: "build", 3: "other", 4: "agg", 5: "masked"}
    dom = max(cls_ms, key=lambda c: cls_ms[c])
    pk = peaks()
    hbm_peak = pk.get("hbm_gbs", 6650.0)
    achieved = cls_bytes[dom] / (cls_ms[dom] / 1e3) / 1e9
    step_bytes = sum(cls_bytes.values())
    # measured DRAM traffic per launch of this kernel class: ncu launch list of the
    # bench command (tools/ncu_traffic.py -> profiles/r2z_traffic.json)
    traffic = None
    try:  # per class: ncu DRAM bytes / ncu device time of the same kernels (64-byte gather granules included)
        trc = json.load(open(os.path.join(ROOT, "profiles", "r2z_traffic.json")))["classes"]
    except Exception:
        trc = {}
    try:
        tr = trc[tclass[dom]]
        traffic = {"dram_bytes_per_launch": tr["dram_bytes_per_launch"],
                   "algorithmic_bytes_per_launch": round(cls_bytes[dom] / cls_n[dom]),
                   "source": "ncu dram__bytes_read.sum + dram__bytes_write.sum, profiles/r2z_traffic.json"}
    except Exception:
        pass
    roofline = {"bound": "hbm", "kernel": names[dom], "achieved": round(achieved, 1),
                "peak": hbm_peak, "unit": "GB/s", "frac": round(achieved / hbm_peak, 4), "traffic": traffic,
                "launches_per_step": cls_n[dom], "share_of_step": round(cls_ms[dom] / sum(cls_ms.values()), 3),
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)" if "hbm_gbs" in pk else "fallback 6.65 TB/s",
                "step_model_gb": round(step_bytes / 1e9, 3),
                "step_gbs": round(step_bytes / (ms_per_step / 1e3) / 1e9 * ws, 1),
                # every kernel class of the step, same event-timed replay and byte model
                "classes": {tclass[c]: dict({"launches_per_step": cls_n[c], "us_per_step": round(cls_ms[c] * 1e3, 1),
                                             "achieved_gbs": round(cls_bytes[c] / (cls_ms[c] / 1e3) / 1e9, 1),
                                             "frac": round(cls_bytes[c] / (cls_ms[c] / 1e3) / 1e9 / hbm_peak, 4),
                                             "share_of_step": round(cls_ms[c] / sum(cls_ms.values()), 3)},
                                            **({"ncu_dram_gbs": round(trc[tclass[c]]["dram_bytes_per_launch"]
                                                                      / trc[tclass[c]]["us_per_launch"] / 1e3, 1),
                                                "ncu_dram_frac": round(trc[tclass[c]]["dram_bytes_per_launch"]
                                                                       / trc[tclass[c]]["us_per_launch"] / 1e3
                                                                       / hbm_peak, 3)}
                                               if tclass[c] in trc else {}))
                            for c in sorted(cls_ms, key=lambda c: -cls_ms[c]) if cls_ms[c] > 0}}

    # ---- e2e through the public API with host buffers: cold cache, every column
    #      H2D from pinned host memory inside the timed region (GPU-only placement)
    # the hot database is done: free its cache and heap before the cold one opens
    # (at SF100 both would not fit one GPU)
    for p in preps:
        p.close()
    db.close()
    torch.cuda.synchronize()

    e2e = None
    e2e_results = None
    if not args.no_e2e:
        cold = Database(device=local, cache_bytes=64 << 30, heap_bytes=heap, placement=A.PLACE_GPU_ONLY,
                        prefetch=not args.no_prefetch)
        load_ssb(cold, shard, row_begin=b, row_end=e, cache=False, presliced=True)
        plans = [ssb_plan(cold, q) for q in SSB_QUERIES]
        all_cols = [(t, c) for (t, c) in cold._cols]

        from paper_conf_sigmod_bressft16_b200.dist import merge_finalized
        roots = [pl.plan.ops[pl.n - 1] for pl in plans]

        def e2e_step():  # the 13 queries submitted at once (the paper's parallel users)
            qs = [cold.submit(pl) for pl in plans]
            res = [cold.fetch(q) for q in qs]
            for (t, c) in all_cols:
                cold.evict(t, c)
            if ws == 1:
                return {q: r.rows for q, r in zip(SSB_QUERIES, res)}
            # N > 1: every rank's finalised results to rank 0, merged exactly there
            import torch.distributed as dist
            gathered = [None] * ws
            dist.all_gather_object(gathered, [r.rows for r in res])
            if rank != 0:
                return None
            return {q: merge_finalized(roots[i], [g[i] for g in gathered]).rows for i, q in enumerate(SSB_QUERIES)}
        for _ in range(2):  # first cold steps pay one-time driver / allocator set-up
            e2e_step()
        cold.reset_stats()
        if ws > 1:
            import torch.distributed as dist
            dist.barrier()
        t0 = time.perf_counter()
        step_ms = []
        for _ in range(args.e2e_steps):
            ts = time.perf_counter()
            e2e_results = e2e_step()
            step_ms.append(round(1e3 * (time.perf_counter() - ts), 1))
        dt = time.perf_counter() - t0
        st = cold.stats()
        h2d, d2h = st["h2d_bytes"], st["d2h_bytes"]
        if ws > 1:  # the whole job: the slowest rank's time, every rank's bytes
            import torch.distributed as dist
            mx = torch.tensor([dt], dtype=torch.float64, device="cuda")
            sm = torch.tensor([float(h2d), float(d2h)], dtype=torch.float64, device="cuda")
            dist.all_reduce(mx, op=dist.ReduceOp.MAX)
            dist.all_reduce(sm, op=dist.ReduceOp.SUM)
            dt, h2d, d2h = float(mx[0]), int(sm[0]), int(sm[1])
        e2e = {"value": total_rows * args.e2e_steps / dt, "unit": UNIT,
               "h2d_bytes_per_step": h2d // args.e2e_steps,
               "d2h_bytes_per_step": d2h // args.e2e_steps,
               "h2d_gbs": round(h2d / dt / 1e9, 2), "step_ms": step_ms,
               "path": "ddq_submit (13 queries at once) / ddq_fetch, GPU-only placement, empty cache; "
                       "columns copied from pinned host memory (cold cache, P:32)" +
                       ("; streamed cold path: the plans' columns stream in from submit while earlier "
                        "operators compute (prefetch, N1)" if not args.no_prefetch else "; on demand") +
                       ("; N > 1: every rank its own rows, finalised results all-gathered to rank 0 and "
                        "merged exactly (dist.merge_finalized); time = slowest rank" if ws > 1 else "")}
        cold.close()
        if args.dump_results and rank == 0 and e2e_results is not None:
            with open(args.dump_results + ".e2e.json", "w") as f:
                json.dump({q: [list(r) for r in rows] for q, rows in e2e_results.items()}, f)

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        cpu = cpu_baseline(sf_total, 6_000_000)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "int64",
                "data": "synthetic (datagen, seed 0x5EED2016)",
                "config": {"workload": f"SSB SF{sf_total:g}, all 13 queries, hot cache" +
                                       (" (BASELINE configs[2]: lineorder row-sharded)" if ws > 1 else
                                        " (BASELINE configs[1])" if sf_total == 20 else ""),
                           "build_once": ws > 1 and backend == "nccl" and args.build_once,
                           "lineorder_rows": n_lo, "rows_per_gpu": shard_rows, "queries": 13,
                           "parallelism": f"row-sharded x{ws}" if ws > 1 else "1 GPU",
                           "query_streams": max(args.streams, 1),
                           "serial_ms_per_step": round(serial_ms / args.steps, 4) if serial_ms else None,
                           "serial_value": total_rows * args.steps / (serial_ms / 1e3) if serial_ms else None,
                           "l2": f"inputs ({fact_gb:.1f} GB of lineorder columns per GPU) larger than L2 "
                                 f"({l2_mb:.0f} MB); no flush"},
                "queries_per_s": 13 * args.steps / (ms / 1e3),
                "gpu_launches": kernels_per_step * args.steps,
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "setup_s": round(setup_s, 1),
                "checks": {q: len(r) for q, r in results.items()}}
        print(json.dumps(line), flush=True)
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
