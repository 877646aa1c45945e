"""Test-side helpers: golden fixture loading and key construction (no race arithmetic)."""
import json
import os

import numpy as np

import tracegen as tg

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
SHARED = 1 << 63
CLS = {"WARP": 1, "BLOCK": 2, "GRID": 3}


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def gkey(word):
    return int(word)


def skey(block, word):
    return SHARED | (int(block) << 32) | int(word)


def expand_expected(rows):
    out = {}
    for space, block, lo, hi, cls in rows:
        for w in range(lo, hi + 1):
            out[gkey(w) if space == "global" else skey(block, w)] = CLS[cls]
    return out


def listing_trace(case, params, shuffle_seed=None):
    fn = {"listing2": tg.listing2, "listing3": tg.listing3, "listing4": tg.listing4,
          "listing5": tg.listing5}[case]
    return fn(shuffle_seed=shuffle_seed, **params)


def scenario_trace(geom, steps):
    """One event per step, in the given order (batch-sorted only if already monotone)."""
    ev = np.empty(len(steps), dtype=tg.EVENT_DTYPE)
    kinds = {"R": tg.READ, "W": tg.WRITE, "AB": tg.ATOMIC_BLOCK, "AG": tg.ATOMIC_GRID}
    for i, (label, kind, b, w) in enumerate(steps):
        blk, wp, t = int(label[1]), int(label[2]), int(label[3])
        ev[i]["addr"] = 0
        ev[i]["tid"] = blk * geom["block_threads"] + wp * geom["warp_size"] + t
        ev[i]["meta"] = tg.pack_meta(kinds[kind], 2, w, b, 0)
    return tg.Trace("scenario", ev, geom["grid_blocks"], geom["block_threads"], geom["warp_size"], 1, 0)


def as_dict(keys, cls):
    return {int(k): int(c) for k, c in zip(keys, cls)}
