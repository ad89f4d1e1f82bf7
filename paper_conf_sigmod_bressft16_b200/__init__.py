"""B200-native hot path of Bress, Funke & Teubner, "Robust Query Processing in
Co-Processor-accelerated Databases" (SIGMOD'16): column-at-a-time relational
operators (selection, hash build/probe, gather, group-by) as sm_100a kernels
behind the C ABI of include/ddq.h, driven by the paper's data-driven placement and
query chopping.  This package is argument marshalling over libddq.so only.
"""
from ._abi import DDQError, lib  # noqa: F401
from .engine import Cluster, Database, PlanBuilder, Prepared, QueryResult  # noqa: F401

__all__ = ["Cluster", "Database", "PlanBuilder", "Prepared", "QueryResult", "DDQError", "lib"]
