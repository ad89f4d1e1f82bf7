"""Multi-GPU data-driven placement (Sec. 6.3) on one device: a
cluster of two databases (two per-GPU caches, here on the same B200), each holding the
SSB tables.  An empty cluster spreads the queries round robin; Algorithm 1 then fills
each member's cache from the accesses of the queries IT ran; afterwards a
query goes to the member whose cache holds most of its input bytes, and inside it each
operator is placed data-driven.  Pins: every result equals the oracle whatever the
member; the members' caches specialise (different column sets); a re-submitted query
lands where its columns are and runs with fewer host operators than before placement."""
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


def test_cluster_routes_queries_to_their_data():
    from paper_conf_sigmod_bressft16_b200 import Cluster
    from paper_conf_sigmod_bressft16_b200.ssb import SSB_QUERIES, load_ssb, ssb_plan, FACT_COLUMNS
    data = datagen.SSB(0.5)
    ws = sum(data[c].nbytes for c in FACT_COLUMNS)
    cl = Cluster([0, 0], cache_bytes=int(0.45 * ws), heap_bytes=2 << 30)
    for m in cl.members:
        load_ssb(m, data, cache=False)
    db0 = cl.members[0]
    plans = {q: ssb_plan(db0, q) for q in SSB_QUERIES}
    want = {q: oracle.run(data, q) for q in SSB_QUERIES}
    before = {}
    for q in SSB_QUERIES:  # empty caches: round robin, every operator on the host
        m, h = cl.submit(plans[q])
        r = cl.fetch(m, h)
        assert r.rows == want[q], q
        before[q] = (m, r.host_ops)
    assert {m for m, _ in before.values()} == {0, 1}
    cl.update_placement()
    cached = [{c for c in m._cols if m.is_cached(*c)} for m in cl.members]
    assert cached[0] and cached[1] and cached[0] != cached[1]  # the caches specialise
    moved_to_gpu = 0
    for q in SSB_QUERIES:
        m, h = cl.submit(plans[q])
        r = cl.fetch(m, h)
        assert r.rows == want[q], q
        # routed to the member holding the most of its input bytes
        in_cols = {(t, c) for (t, c) in db0._cols if c in _plan_columns(db0, plans[q])}
        held = [sum(data[c].nbytes for (t, c) in in_cols if (t, c) in cached[i]) for i in range(2)]
        assert held[m] == max(held), (q, held, m)
        moved_to_gpu += r.host_ops < before[q][1]
    assert moved_to_gpu > 0
    cl.close()


def _plan_columns(db, P):
    """Names of the columns a plan reads (from the plan structs)."""
    ids = set()
    for i in range(P.n):
        op = P.plan.ops[i]
        for k in range(op.n_preds):
            ids.add(op.preds[k].column)
        for c in (op.key_col, op.payload_col, op.fk_col, op.gather_col):
            if c >= 0:
                ids.add(c)
        for k in range(op.n_keys):
            if op.key_src[k] < -1:
                ids.add(-2 - op.key_src[k])
        for a in range(op.n_aggs):
            for j in range(3):
                if op.agg_col[a][j] >= 0:
                    ids.add(op.agg_col[a][j])
        for j in range(op.n_terms):
            ids.add(op.term_fk[j])
    names = {v: c for (t, c), v in db._cols.items()}
    return {names[i] for i in ids if i in names}
