"""C-ABI checks that need no GPU: libddq.so loads, exports every entry point that
include/ddq.h declares, the ctypes binding's struct layouts equal the C layouts,
and the product path refuses to run without a CUDA device (no CPU fallback)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ddq.h")


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(ddq_[a-z0-9_]+)\s*\(", text)))


def test_library_exports_every_declared_symbol():
    from paper_conf_sigmod_bressft16_b200 import _abi
    L = _abi.lib()
    names = declared_functions()
    assert len(names) > 40
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing
    # and the binding covers all of them
    assert set(names) == set(_abi.SIGNATURES), set(names) ^ set(_abi.SIGNATURES)


def test_so_is_sm100a():
    so = os.path.join(ROOT, "paper_conf_sigmod_bressft16_b200", "libddq.so")
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", so], capture_output=True, text=True).stdout
    assert "sm_100a" in out


LAYOUT_C = r"""
#include <stdio.h>
#include <stddef.h>
#include "ddq.h"
#define P(T) printf(#T " %zu\n", sizeof(T));
#define O(T, f) printf(#T "." #f " %zu\n", offsetof(T, f));
int main(void) {
  P(ddq_dev_pred) P(ddq_dev_agg) P(ddq_config) P(ddq_pred) P(ddq_op) P(ddq_plan) P(ddq_result) P(ddq_stats)
  O(ddq_op, preds) O(ddq_op, key_col) O(ddq_op, agg_col) O(ddq_op, max_groups) O(ddq_op, order_by)
  O(ddq_op, limit) O(ddq_config, cache_bytes) O(ddq_config, fault_alloc_every) O(ddq_result, exec_ms)
  O(ddq_dev_pred, in_vals) O(ddq_dev_agg, arg) O(ddq_op, eq_cmp) O(ddq_op, build_key_set)
  O(ddq_op, n_avg) O(ddq_op, avg_scale) O(ddq_result, agg_null) O(ddq_result, avgs) O(ddq_result, key_str)
  O(ddq_op, gather_narrow) O(ddq_result, op_place) O(ddq_config, fault_op_mask) O(ddq_result, op_ms) O(ddq_config, prefetch)
  O(ddq_config, placement_period_ms) O(ddq_config, max_queries)
  printf("DDQ_CMP_EQ %d\nDDQ_CMP_LT %d\nDDQ_CMP_NE %d\nDDQ_AGG_MIN %d\nDDQ_AGG_COUNT %d\n",
         DDQ_CMP_EQ, DDQ_CMP_LT, DDQ_CMP_NE, (int)DDQ_AGG_MIN, (int)DDQ_AGG_COUNT);
  printf("DDQ_PRED_BITSET %d\n", (int)DDQ_PRED_BITSET);
  return 0;
}
"""


def test_struct_layouts_match_c(tmp_path):
    from paper_conf_sigmod_bressft16_b200 import _abi as A
    src = tmp_path / "layout.c"
    src.write_text(LAYOUT_C)
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = dict(line.split() for line in subprocess.check_output([str(exe)], text=True).splitlines())
    py = {"ddq_dev_pred": A.DevPred, "ddq_dev_agg": A.DevAgg, "ddq_config": A.Config, "ddq_pred": A.Pred,
          "ddq_op": A.Op, "ddq_plan": A.Plan, "ddq_result": A.Result, "ddq_stats": A.Stats}
    consts = {"DDQ_CMP_EQ": A.CMP_EQ, "DDQ_CMP_LT": A.CMP_LT, "DDQ_CMP_NE": A.CMP_NE,
              "DDQ_AGG_MIN": A.AGG_MIN, "DDQ_AGG_COUNT": A.AGG_COUNT, "DDQ_PRED_BITSET": A.PRED_BITSET}
    for k, v in got.items():
        if k in consts:
            assert consts[k] == int(v), k
        elif "." in k:
            t, f = k.split(".")
            assert getattr(py[t], f).offset == int(v), k
        else:
            assert ctypes.sizeof(py[k]) == int(v), k


def test_open_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_sigmod_bressft16_b200 import Database, DDQError
    with pytest.raises(DDQError) as e:
        Database()
    assert "DDQ_ECUDA" in str(e.value)


def test_version_string():
    from paper_conf_sigmod_bressft16_b200 import _abi
    assert b"sm_100a" in _abi.lib().ddq_version()
