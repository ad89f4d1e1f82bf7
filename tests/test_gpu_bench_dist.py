"""bench.py's N>1 path end to end on one GPU: two ranks (torchrun, gloo backend
through the DDQ_BENCH_BACKEND test hook, both on cuda:0) each run the 13 prepared
plans on their half of lineorder, exchange the compacted partial group tables and
rank 0 merges them -- the merged results equal the oracle on the whole table
(S8(e): sharding and the exchange never change results); the end-to-end path (every
rank cold-loads its rows and runs the 13 queries through ddq_submit, rank 0 merges
the finalised results) equals it too."""
import json
import os
import subprocess
import sys

import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_two_ranks_merged_results_equal_oracle(tmp_path):
    out = tmp_path / "results.json"
    env = dict(os.environ, DDQ_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29533", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--sf", "0.25", "--steps", "3", "--warmup", "3", "--e2e-steps", "1", "--no-cpu-baseline",
           "--dump-results", str(out)]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    got = json.load(open(out))
    cold = json.load(open(str(out) + ".e2e.json"))  # the end-to-end path: ddq_submit per rank, merged
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 2 and line["e2e"]["value"] > 0 and line["e2e"]["h2d_bytes_per_step"] > 0
    data = datagen.SSB(0.5)  # 2 ranks x SF 0.25
    for q in oracle.SSB_QUERIES:
        want = [list(x) for x in oracle.run(data, q)]
        g = got[q]
        if q.startswith("ssb1") and not g:
            want = [w for w in want if w != [0, 0]]
        assert g == want, q
        assert cold[q] == [list(x) for x in oracle.run(data, q)], q
