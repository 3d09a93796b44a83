"""CPU checks of the C-ABI boundary: libtsv.so loads and exports every symbol include/*.h declares;
host-only calls (index maps, presets, argument errors) work without a GPU."""
import os
import re

import numpy as np
import pytest

from oracle import sp as SP

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = set()
    for h in ("tsv.h", "tsv_ops.h", "tsv_sched.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        names |= set(re.findall(r"\b(tsv_[a-z_0-9]+)\s*\(", src))
    return names


@pytest.fixture(scope="module")
def tsv():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_asplos_luhtlwm0c26_b200 as m
    return m


def test_exports_every_declared_symbol(tsv):
    declared = _declared()
    assert len(declared) >= 30
    for name in declared:
        assert hasattr(tsv.lib, name), name
    assert declared == set(tsv.EXPORTED)


def test_shard_range_matches_oracle_index_map(tsv):
    for n in (0, 1, 7, 64, 333, 1024, 16384):
        for k in (1, 2, 4, 8):
            for r in range(k):
                assert tsv.shard_range(n, k, r) == SP.shard_range(n, k, r)


def test_reshard_plan_matches_oracle(tsv):
    for n in (5, 1024, 1037, 16384):
        for ks in (1, 2, 4, 8):
            for kd in (1, 2, 4, 8):
                assert tsv.reshard_plan(n, ks, kd) == SP.reshard_plan(n, ks, kd)


def test_presets_and_errors(tsv):
    d = tsv.model_preset("flux")
    assert (d.hidden, d.heads, d.head_dim, d.mlp_hidden, d.n_double, d.n_single, d.text_tokens) == \
        (3072, 24, 128, 12288, 19, 38, 512)
    assert list(d.axes_dim) == [16, 56, 56]
    with pytest.raises(tsv.TsvError) as ei:
        tsv.model_preset("nope")
    assert ei.value.status == -1
    with pytest.raises(tsv.TsvError):
        tsv.shard_range(10, 0, 0)
    with pytest.raises(tsv.TsvError):
        tsv.shard_range(10, 2, 2)


def test_sd3_presets(tsv):
    d = tsv.model_preset("sd3")
    assert (d.hidden, d.heads, d.head_dim, d.mlp_hidden, d.n_double, d.n_single, d.text_tokens, d.vec_dim) == \
        (1536, 24, 64, 6144, 24, 0, 333, 2048)
    assert d.family == 1 and d.cfg_scale == 7.0 and d.shift == 3.0 and (d.pe_max, d.pe_base) == (192, 64)
    t = tsv.model_preset("tiny_sd3")
    assert (t.hidden, t.heads, t.n_double, t.text_tokens, t.family) == (256, 4, 2, 77, 1)
    assert tsv.model_preset("flux").family == 0
