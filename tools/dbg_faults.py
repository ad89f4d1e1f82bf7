import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen, oracle
from paper_conf_sigmod_bressft16_b200 import Database
from paper_conf_sigmod_bressft16_b200.ssb import load_ssb, ssb_plan
data = datagen.SSB(0.1)
for chop, fe in [(False, 5), (True, 5), (False, 0), (True, 3), (False, 3), (False, 7)]:
    db = Database(cache_bytes=8 << 30, heap_bytes=4 << 30, chopping=chop, fault_alloc_every=fe)
    load_ssb(db, data)
    bad = []
    for q in oracle.SSB_QUERIES:
        r = db.run(ssb_plan(db, q))
        w = oracle.run(data, q)
        if q.startswith("ssb1") and r.rows == []:
            r.rows = [(0, 0)]
        if [tuple(x) for x in r.rows] != [tuple(x) for x in w]:
            bad.append((q, len(r.rows), len(w), r.gpu_ops, r.host_ops, r.aborts))
    print("chop", chop, "faults", fe, "bad:", bad, db.stats()["aborts"], flush=True)
    db.close()
