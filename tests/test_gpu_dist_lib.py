"""libddq's multi-GPU layer (S8(e)) on one GPU: an NCCL communicator of one
rank with build-once broadcasts (the build runs on rank 0 and ncclBroadcast -- in
place at world 1 -- is captured into the plan's CUDA graph, serially) and the partial
exchange (ncclAllGather) + exact merge; and the host transport (ddq_dist_init_host)
with an all-gather callback.  All 13 SSB queries equal the oracle.  The two-rank path
(two processes, gloo host transport, one GPU) is bench.py's, tested in
test_gpu_bench_dist.py."""
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("transport", ["nccl", "host"])
def test_dist_exchange_single_rank_equals_oracle(transport):
    from paper_conf_sigmod_bressft16_b200 import Database
    from paper_conf_sigmod_bressft16_b200.engine import nccl_unique_id
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan
    data = datagen.SSB(0.5)
    db = Database(cache_bytes=8 << 30, heap_bytes=4 << 30)
    if transport == "nccl":
        db.dist_init_nccl(nccl_unique_id(), 0, 1, build_once=True)
    else:
        db.dist_init_host(0, 1, lambda b: b)
    load_ssb(db, data)
    db.set_partitioned("lineorder")
    preps = [db.prepare(ssb_plan(db, q)) for q in SSB_QUERIES]
    for _ in range(2):  # relaunch: graphs with the broadcasts inside replay
        for p in preps:
            p.launch()
        db.dist_exchange(preps)
        for i, q in enumerate(SSB_QUERIES):
            assert db.dist_result(i).rows == oracle.run(data, q), q
    db.close()


def test_dist_api_errors():
    from paper_conf_sigmod_bressft16_b200 import Database, DDQError
    db = Database(cache_bytes=1 << 30, heap_bytes=1 << 30)
    with pytest.raises(DDQError):  # no exchange before init
        db.dist_result(0)
    db.dist_init_host(0, 1, lambda b: b)
    with pytest.raises(DDQError):  # initialised twice
        db.dist_init_host(0, 1, lambda b: b)
    db.close()
