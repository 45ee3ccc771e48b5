"""Per-shape tile search results: the paper's "auto-search ... through profile runs" (P:L271-273,
section 5.1), whose outcome "only need[s] to be determined once per convolution shape".

qconv_autotune (include/qconv.h) times every candidate plan of one descriptor on the GPU and
records the fastest for that descriptor in the library's process-wide plan table.  This module
only persists that table: a JSON list of {descriptor fields, chosen kernel / N tile, time}
entries, written after a search and applied with qconv_plan_set when loaded.  No computation
of the method happens here.
"""
from __future__ import annotations

import json
import os
from typing import Iterable, List

from . import (KERNEL_NAMES, qconv_autotune, qconv_debug_plan, qconv_desc, qconv_plan_set)

_FIELDS = [f for f, _ in qconv_desc._fields_ if f != "w_zero"]


def desc_fields(d: qconv_desc) -> dict:
    out = {f: int(getattr(d, f)) for f in _FIELDS}
    out["w_zero"] = 1 if d.w_zero else 0
    return out


def desc_from_fields(f: dict) -> qconv_desc:
    d = qconv_desc()
    for k in _FIELDS:
        setattr(d, k, int(f[k]))
    return d


def tune_layers(layers: Iterable[dict], iters: int = 5) -> List[dict]:
    """layers: dicts with desc, x, w, bias, m, n, y (device tensors, as bench.Trunk holds them).
    Runs the profile-run search for each and returns the table entries."""
    entries = []
    for L in layers:
        best, us = qconv_autotune(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"],
                                  iters=iters)
        entries.append({"name": L.get("name", ""), "desc": desc_fields(L["desc"]),
                        "kernel": best["kernel"], "kernel_name": KERNEL_NAMES[best["kernel"]],
                        "bn": best["bn"], "us": us})
    return entries


def save_plans(path: str, entries: List[dict], meta: dict = None) -> None:
    with open(path, "w") as f:
        json.dump({"meta": meta or {}, "plans": entries}, f, indent=1)


def load_plans(path: str) -> int:
    """Apply every entry of a saved table (qconv_plan_set); entries whose descriptor w_zero is
    set are skipped (the table does not hold device pointers).  Returns how many were applied."""
    if not os.path.exists(path):
        return 0
    with open(path) as f:
        data = json.load(f)
    n = 0
    for e in data["plans"]:
        if e["desc"].get("w_zero"):
            continue
        d = desc_from_fields(e["desc"])
        qconv_plan_set(d, e["kernel"], e["bn"])
        assert qconv_debug_plan(d)["kernel"] == e["kernel"]
        n += 1
    return n
