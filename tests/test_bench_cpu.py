"""bench.py's per-config defaults (host logic, no GPU): cache mode and H2D path per config, and
that flags the user gives always win."""
import argparse

import bench


def _args(config, mode=None, copy_method=None, copy_ctas=0, load_priority=None, tier=None):
    return argparse.Namespace(config=config, mode=mode, copy_method=copy_method,
                              copy_ctas=copy_ctas, load_priority=load_priority, tier=tier)


def test_c3_defaults_kv_whole_entry_dma():
    a = bench.resolve_defaults(_args("C3"))
    assert (a.mode, a.copy_method, a.copy_ctas, a.load_priority) == ("kv", 2, 0, 0)


def test_c4_defaults_y_whole_entry_dma():
    a = bench.resolve_defaults(_args("C4"))
    assert (a.mode, a.copy_method, a.load_priority) == ("y", 2, 0)


def test_c4_kv_uses_the_wide_row_gather_on_the_host_tier_only():
    a = bench.resolve_defaults(_args("C4", mode="kv"))
    assert (a.copy_method, a.copy_ctas, a.load_priority) == (3, 8, -5)
    a = bench.resolve_defaults(_args("C4", mode="kv", tier="hbm"))
    assert (a.copy_method, a.load_priority) == (2, 0)


def test_sdxl_levels_default_to_y():
    for c in ("C2A", "C2B"):
        a = bench.resolve_defaults(_args(c))
        assert (a.mode, a.copy_method) == ("y", 2)


def test_flags_win():
    a = bench.resolve_defaults(_args("C4", mode="kv", copy_method=2, load_priority=0))
    assert (a.mode, a.copy_method, a.load_priority) == ("kv", 2, 0)
    a = bench.resolve_defaults(_args("C3", copy_method=3, copy_ctas=6))
    assert (a.copy_method, a.copy_ctas, a.load_priority) == (3, 6, -5)
