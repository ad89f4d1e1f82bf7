"""Microbenchmarks of the scan/star kernels on synthetic columns (CUDA-event timed).

Isolates streaming from compaction: dense select over n int64 / int32 rows with
pass fractions 0, 0.15, 1; dense join-index probe with a small bitmap.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def timeit(fn, reps=10):
    import torch
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    import torch
    only = sys.argv[1] if len(sys.argv) > 1 else ""
    from paper_conf_sigmod_bressft16_b200 import ops
    n = 120_000_000
    g = torch.Generator(device="cuda").manual_seed(1)
    c64 = torch.randint(0, 100, (n,), device="cuda", dtype=torch.int64, generator=g)
    c32 = torch.randint(1, 600_001, (n,), device="cuda", dtype=torch.int32, generator=g)
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    pay = torch.empty(n, dtype=torch.int32, device="cuda")
    cnt = ops.count_cell()
    scratch = torch.empty(ops.lib().ddq_op_scratch_bytes(n), dtype=torch.uint8, device="cuda")
    import ctypes
    from paper_conf_sigmod_bressft16_b200 import _abi as A

    def sel(col, lo, hi):
        dp = ops._dev_preds([(col, lo, hi)])
        return lambda: ops.check(ops.lib().ddq_op_select(dp, 1, None, None, n, None, None, 0, out.data_ptr(),
                                                         cnt.data_ptr(), scratch.data_ptr(), scratch.numel(),
                                                         ops._stream()))
    for name, col, lo, hi in [("i64 pass 0", c64, 1000, 2000), ("i64 pass 15%", c64, 0, 14),
                              ("i64 pass 100%", c64, 0, 100), ("i32 pass 0", c32, -5, -1),
                              ("i32 pass 20%", c32, 1, 120000)]:
        if only and only not in "select " + name:
            continue
        ms = timeit(sel(col, lo, hi))
        gb = n * col.element_size() / 1e9
        print(f"select {name:14s} {ms*1e3:8.1f} us  {gb/ms*1e3:8.1f} GB/s (input only)", flush=True)
    for small in (2556, 40_000, 600_000):
        if only and only != "small":
            break
        ms = timeit(lambda: ops.check(ops.lib().ddq_op_select(ops._dev_preds([(c32, 1, 120000)]), 1, None, None, small,
                                                               None, None, 0, out.data_ptr(), cnt.data_ptr(),
                                                               scratch.data_ptr(), scratch.numel(), ops._stream())),
                    reps=50)
        print(f"select i32 n={small:8d} {ms*1e3:8.1f} us", flush=True)
    for rng_keys, frac in ((600_000, 0.2), (600_000, 0.05), (1_000_000, 0.04)):
        fk = c32 if rng_keys == 600_000 else torch.randint(1, rng_keys + 1, (n,), device="cuda", dtype=torch.int32,
                                                           generator=g)
        keys = torch.arange(1, rng_keys + 1, dtype=torch.int32, device="cuda")
        sel_rows = torch.nonzero(torch.rand(rng_keys, device="cuda", generator=g) < frac).int().flatten()
        idx, err = ops.join_index_build(keys, 1, rng_keys, payload=keys, in_tids=sel_rows,
                                        in_count=ops.count_cell(sel_rows.numel()), n=sel_rows.numel())
        for emit in (False, True):
            tag = f"probe bitmap{(rng_keys + 7) // 8 // 1024}KB pass {frac:.2f} emit={emit}"
            if only and only not in tag:
                continue

            def probe():
                ops.check(ops.lib().ddq_op_join_index_probe(idx.data_ptr(), 1, rng_keys, fk.data_ptr(), None, None,
                                                            n, None, None, 0, out.data_ptr(),
                                                            pay.data_ptr() if emit else None, cnt.data_ptr(),
                                                            scratch.data_ptr(), scratch.numel(), ops._stream()))
            ms = timeit(probe)
            print(f"probe  bitmap{(rng_keys + 7) // 8 // 1024}KB pass {frac:.2f} emit={emit} {ms*1e3:8.1f} us"
                  f"  {n*4/1e9/ms*1e3:8.1f} GB/s", flush=True)
    if only:
        return
    ms = timeit(lambda: out.copy_(c32))
    print(f"torch copy int32 (read+write) {ms*1e3:8.1f} us  {2*n*4/1e9/ms*1e3:8.1f} GB/s")


if __name__ == "__main__":
    main()
