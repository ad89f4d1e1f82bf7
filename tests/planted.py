"""A tiny SSB database with planted rows so that every SSB query has matches.

Used to pin the oracle with a pure-Python nested-loop brute force and SQLite.
Plants are written as dictionary codes looked up from the decoded strings, so a
wrong dictionary would show up as a mismatch against the brute force (which works
on strings).
"""
from __future__ import annotations

import numpy as np

import datagen


class Planted(dict):
    """dict column -> array, with the SSB accessors the oracle wrapper uses."""

    def __init__(self, sf=0.002, seed=datagen.DEFAULT_SEED, n_planted=400):
        super().__init__()
        base = datagen.SSB(sf, seed)
        for cols in datagen.SSB_COLUMNS.values():
            for c in cols:
                self[c] = base[c].copy()
        self.sf = sf
        code = {d: {s: i for i, s in enumerate(datagen.dictionary(d))} for d in datagen.DICTS}

        def city(nation_name, digit):
            return (nation_name[:9].ljust(9) + str(digit))

        def plant_geo(prefix, row, nation, region, digit):
            self[prefix + "_city"][row] = code["city"][city(nation, digit)]
            self[prefix + "_nation"][row] = code["nation"][nation]
            self[prefix + "_region"][row] = code["region"][region]

        geos = [("UNITED KINGDOM", "EUROPE", 1), ("UNITED KINGDOM", "EUROPE", 5),
                ("UNITED STATES", "AMERICA", 3), ("CHINA", "ASIA", 2)]
        for r, g in enumerate(geos):
            plant_geo("s", r, *g)
        cgeos = [("UNITED KINGDOM", "EUROPE", 1), ("UNITED KINGDOM", "EUROPE", 5),
                 ("UNITED STATES", "AMERICA", 7), ("JAPAN", "ASIA", 1)]
        for r, g in enumerate(cgeos):
            plant_geo("c", r, *g)
        parts = [("MFGR#1", "MFGR#12", "MFGR#1215"), ("MFGR#2", "MFGR#22", "MFGR#2225"),
                 ("MFGR#2", "MFGR#22", "MFGR#2239"), ("MFGR#1", "MFGR#14", "MFGR#147"),
                 ("MFGR#2", "MFGR#21", "MFGR#2110")]
        for r, (m, c, b) in enumerate(parts):
            self["p_mfgr"][r] = code["mfgr"][m]
            self["p_category"][r] = code["category"][c]
            self["p_brand1"][r] = code["brand1"][b]
        dates = [19971215, 19930610, 19940105, 19940208, 19980301]
        for i in range(n_planted):
            self["lo_custkey"][i] = 1 + i % 4
            self["lo_suppkey"][i] = 1 + (i // 4) % 4
            self["lo_partkey"][i] = 1 + (i // 16) % 5
            self["lo_orderdate"][i] = dates[(i // 80) % 5]
            self["lo_discount"][i] = i % 11
            self["lo_quantity"][i] = (i * 7) % 50 + 1

    def dict_for(self, col):
        return datagen.dictionary(datagen.SSB_STRING_COLUMNS[col])

    def rows(self, table):
        return len(self[datagen.SSB_COLUMNS[table][0]])
