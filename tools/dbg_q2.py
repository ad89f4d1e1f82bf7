"""Debug: TPC-H Q2 on sparse keys through the chopping driver, printing the error
cell after every GPU operator (DDQ_DEBUG_ERRORS=1)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["DDQ_DEBUG_ERRORS"] = "1"
import datagen  # noqa: E402
from paper_conf_sigmod_bressft16_b200 import Database  # noqa: E402
from paper_conf_sigmod_bressft16_b200.tpch import load_tpch, tpch_plan  # noqa: E402

data = datagen.TPCH(float(sys.argv[1]) if len(sys.argv) > 1 else 1, keys="sparse")
db = Database(cache_bytes=8 << 30, heap_bytes=8 << 30)
load_tpch(db, data)
try:
    print(len(db.run(tpch_plan(db, "tpch2")).rows))
except Exception as e:
    print("ERR", e)
