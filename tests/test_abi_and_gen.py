"""Host-side checks (-m "not gpu"): the C-ABI library loads and exports every symbol the header
declares; the shared input generators are deterministic and host/indexed variants agree."""
import ctypes
import os
import re
import subprocess

import numpy as np

import gen
from gen import configs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    hdr = open(os.path.join(ROOT, "include", "spade.h")).read()
    return sorted(set(re.findall(r"SPADE_API\s+[\w\s\*]+?\b(spade_\w+)\s*\(", hdr)))


def test_header_declares_the_survey_entry_points():
    syms = _declared_symbols()
    for s in ("spade_build_canvas", "spade_select", "spade_join_count", "spade_join_pairs"):
        assert s in syms


def test_library_builds_loads_and_exports_every_declared_symbol():
    from paper_conf_icde_doraiswamyf22_b200 import build as b
    lib_path = b.build()
    out = subprocess.run(["nm", "-D", "--defined-only", lib_path], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (spade_\w+)", out))
    assert set(_declared_symbols()) <= exported
    lib = ctypes.CDLL(lib_path)                     # loads without a GPU (lazy CUDA init)
    for s in _declared_symbols():
        getattr(lib, s)
    import paper_conf_icde_doraiswamyf22_b200 as sp
    assert set(sp.EXPORTED_SYMBOLS) == set(_declared_symbols())
    lib.spade_status_string.restype = ctypes.c_char_p
    assert lib.spade_status_string(-3) == b"output capacity too small"


def test_point_generator_is_deterministic_and_indexable():
    tp = gen.taxi_params(301)
    a = gen.points_host(tp, 301, 1000, 5000)
    b = gen.points_host(tp, 301, 1000, 5000)
    assert np.array_equal(a, b)
    idx = np.array([1000, 1001, 5999, 3333], np.int64)
    assert np.array_equal(gen.points_at(tp, 301, idx), a[idx - 1000])
    assert a.min() >= 0 and a.max() < gen.DOMAIN
    u = gen.points_host(gen.uniform_params(0, 0, 1024, 1024), 101, 0, 10000)
    assert u.min() >= 0 and u.max() < 1024


def test_taxi_points_are_clustered():
    """Zipf head: the most popular 1/64 of the domain holds far more than 1/64 of the points."""
    tp = gen.taxi_params(301)
    xy = gen.points_host(tp, 301, 0, 200_000)
    cell = (xy[:, 1] >> 21) * 8 + (xy[:, 0] >> 21)
    h = np.bincount(cell, minlength=64) / len(xy)
    assert h.max() > 5 / 64


def test_config_polygon_sets_have_the_stated_shapes():
    c3 = configs.c3(10).polys
    assert len(c3["poly_ring_off"]) - 1 == 260 and len(c3["ring_xy"]) == 260 * 540
    c4 = configs.c4(10).polys
    assert len(c4["poly_ring_off"]) - 1 == 50 * 42 + 100
    c2 = configs.c2(10).polys
    assert len(c2["ring_xy"]) == 1000


def test_set_option_validates_names_and_values_without_a_gpu():
    """spade_set_option (probe-path tuning, include/spade.h) is host-only: valid settings are
    accepted, unknown names and out-of-range values are INVALID_ARG."""
    import paper_conf_icde_doraiswamyf22_b200 as sp
    lib = sp.load()
    for name, value in [("defer", 1), ("defer", 0), ("coop", 8), ("coop", -1), ("cache_slots", 4096),
                        ("cache_slots", 16384), ("count_global", 0), ("global_queue", 0), ("debug_defer", 0), ("pipe", 1), ("pipe", -1),
                        ("hist_copies_max", 1), ("hist_copies_max", 16), ("idx_queue", 1), ("idx_queue", 0), ("idx_queue", -1)]:
        assert lib.spade_set_option(name.encode(), value) == 0, name
    for name, value in [("coop", 3), ("cache_slots", 1000), ("defer", 2), ("pipe", 2), ("nope", 0),
                        ("hist_copies_max", 64), ("hist_copies_max", 12), ("idx_queue", 2)]:
        assert lib.spade_set_option(name.encode(), value) == -1, name
    assert lib.spade_set_option(None, 0) == -1
