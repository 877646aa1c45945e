"""Compact 4-byte shadow records (include/hirace.h hirace_shadow_alloc_compact;
PAPER.md L289 "8 bytes of memory per address by default (though this is configurable and can
be reduced)", L419-423 "removing memory allocated for clocks in those programs that do not
utilize synchronization").  CPU only, through the C-ABI verification hook
hirace_fsm_step_compact (the compact replay kernels' own label/next functions and raw table):

* isomorphism with the 8-byte automaton: on every step of random tiny traces x random linear
  extensions, the compact record holds exactly the 8-byte record's fields, and the report
  flags agree;
* the compact automaton against the literal brute-force enumerator (race set + class);
* layout: field widths follow the declared limits; a layout wider than 32 bits is refused;
  epochs the program does not use take no bits (the paper's "no synchronization" case).
"""
import numpy as np
import pytest

import tracegen as tg
from oracle import brute

h = pytest.importorskip("paper_conf_sc_jacobsonbg24_b200")

from tests.test_fsm import _random_linear_extension, _unpack  # noqa: E402


def _bits(x):
    return int(x).bit_length()


def _layout(lim, threads):
    gb, bb, wb = (_bits(v) for v in lim)
    sh_b = 5 + gb
    sh_w = sh_b + bb
    sh_t = sh_w + wb
    return sh_b, sh_w, sh_t, max(1, _bits(threads - 1))


def _to_compact(o64, lim, threads):
    """The 8-byte record's fields repacked in the compact layout (an independent restatement of
    include/hirace.h's field list, used only to compare the two automata)."""
    sh_b, sh_w, sh_t, _ = _layout(lim, threads)
    st, g, b, w, tid = o64 & 31, (o64 >> 5) & 255, (o64 >> 13) & 1023, (o64 >> 23) & 511, o64 >> 32
    return st | (g << 5) | (b << sh_b) | (w << sh_w) | (tid << sh_t)


def _limits(acc):
    return (max(a["g"] for a in acc), max(a["b"] for a in acc), max(a["w"] for a in acc))


@pytest.mark.parametrize("policy", [0, 1])
@pytest.mark.parametrize("chunk", range(3))
def test_compact_automaton_is_the_8_byte_automaton(chunk, policy):
    rng = np.random.default_rng(7000 + chunk + 10 * policy)
    steps = 0
    for seed in range(chunk * 300, (chunk + 1) * 300):
        t = tg.random_tiny(seed)
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        threads = t.grid_blocks * t.block_threads
        lim = _limits(acc)
        for _ in range(2):
            order = _random_linear_extension(acc, rng)
            s64, s32 = {}, {}
            for i in order:
                a = acc[i]
                o64, o32 = s64.get(a["key"], 0), s32.get(a["key"], 0)
                n64, r64 = h.fsm_step(o64, a["tid"], a["kind"], a["g"], a["b"], a["w"], t.block_threads,
                                      t.warp_size, policy=policy)
                n32, r32 = h.fsm_step_compact(o32, a["tid"], a["kind"], a["g"], a["b"], a["w"], t.block_threads,
                                              t.warp_size, threads, lim, policy=policy)
                assert n32 == _to_compact(n64, lim, threads), (seed, a, hex(n64), hex(n32))
                assert r32 == r64
                s64[a["key"]], s32[a["key"]] = n64, n32
                steps += 1
    assert steps > 5000


@pytest.mark.parametrize("chunk", range(2))
def test_compact_bisimulation_vs_brute_force(chunk):
    rng = np.random.default_rng(9100 + chunk)
    for seed in range(5000 + chunk * 400, 5000 + (chunk + 1) * 400):
        t = tg.random_tiny(seed)
        want = {k: c for k, (c, _) in brute.races(t.events, t.block_threads, t.warp_size).items()}
        acc = _unpack(t.events, t.block_threads, t.warp_size)
        threads = t.grid_blocks * t.block_threads
        lim = _limits(acc)
        for _ in range(3):
            shadow = {}
            for i in _random_linear_extension(acc, rng):
                a = acc[i]
                shadow[a["key"]], _ = h.fsm_step_compact(shadow.get(a["key"], 0), a["tid"], a["kind"], a["g"],
                                                         a["b"], a["w"], t.block_threads, t.warp_size, threads, lim)
            got = {k: (v & 31) - 19 for k, v in shadow.items() if (v & 31) >= 20}
            assert got == want, seed


def test_layout_widths_and_refusal():
    # sync-free program (only kernel boundaries): no b / w bits; 2^20 threads, 31 grid epochs
    n, _ = h.fsm_step_compact(0, (1 << 20) - 1, 1, 31, 0, 0, 256, 32, 1 << 20, (31, 0, 0))
    assert n & 31 == 4 and n >> 10 == (1 << 20) - 1 and (n >> 5) & 31 == 31
    # 2^24 threads + 4 g + 4 b + 2 w epochs (config 5) needs 5+2+2+1+24 = 34 bits: refused
    n, _ = h.fsm_step_compact(0, 0, 1, 0, 0, 0, 256, 32, 1 << 24, (3, 3, 1))
    assert n == 0xFFFFFFFF
    # exactly 32 bits fits: 5 + 8 + 0 + 0 + 19
    n, _ = h.fsm_step_compact(0, (1 << 19) - 1, 0, 200, 0, 0, 256, 32, 1 << 19, (255, 0, 0))
    assert n != 0xFFFFFFFF and n >> 13 == (1 << 19) - 1 and (n >> 5) & 255 == 200


@pytest.mark.parametrize("name,make,lim_bits", [
    ("cfg2", lambda: tg.cfg2(True, n=64, steps=8), 32),
    ("cfg4", lambda: tg.cfg4("G", 8, 128, 34), 32),
    ("cfg3", lambda: tg.cfg3("bfs", True, scale=10), 32),
])
def test_paper_shaped_configs_fit_compact(name, make, lim_bits):
    """configs 1-4 fit the compact record at their bench sizes (thread counts from BASELINE.json
    configs; epoch maxima from the generators); config 5 (2^24 threads) does not."""
    t = make()
    lim = h.trace_epoch_limits(t.events)
    full_threads = {"cfg2": 1024 * 256, "cfg4": 592 * 256, "cfg3": 4096 * 256}[name]
    sh_b, sh_w, sh_t, tb = _layout(lim, full_threads)
    assert sh_t + tb <= lim_bits, (name, lim, sh_t, tb)
