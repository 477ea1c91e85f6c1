"""The oracle pins have teeth: plausible one-line slips in the oracle must fail them (-m "not gpu").

Each mutant is a copy of oracle/spade_oracle.c with one edit, compiled into a scratch directory;
tests/test_oracle_pins.py is then run against it in a subprocess and must report failures.
"""
import os
import shutil
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

MUTANTS = {
    "tie_rule_counts_o_eq_0": ("return by > ay ? (o > 0) : (o < 0);", "return (o > 0) == (by > ay);"),
    "drop_closing_edge": ("for (int64_t k = v0; k < v1; ++k) {", "for (int64_t k = v0; k + 1 < v1; ++k) {"),
    "closed_straddle": ("if ((ay > py) == (by > py)) return 0;", "if ((ay >= py) == (by >= py)) return 0;"),
    "transposed_operand": ("__int128 o = (__int128)(bx - ax) * (py - ay) - (__int128)(by - ay) * (px - ax);",
                           "__int128 o = (__int128)(by - ay) * (py - ay) - (__int128)(bx - ax) * (px - ax);"),
    "first_ring_only": ("for (int64_t r = ring_begin; r < ring_end; ++r) {",
                        "for (int64_t r = ring_begin; r < ring_begin + 1 && r < ring_end; ++r) {"),
    "flipped_sign": ("return by > ay ? (o > 0) : (o < 0);", "return by > ay ? (o < 0) : (o > 0);"),
}
# distance / kNN oracle (oracle/distance_oracle.c) against tests/test_distance_oracle_pins.py
DIST_MUTANTS = {
    "open_disk": ("return dx * dx + dy * dy <= (__int128)r2;", "return dx * dx + dy * dy < (__int128)r2;"),
    "dropped_dy": ("return dx * dx + dy * dy <= (__int128)r2;", "return dx * dx <= (__int128)r2;"),
    "mixed_term": ("return dx * dx + dy * dy <= (__int128)r2;", "return dx * dx + dx * dy <= (__int128)r2;"),
    "int64_overflow": ("__int128 dx = (__int128)px - cx, dy = (__int128)py - cy;\n    return",
                       "int64_t dx = px - cx, dy = py - cy;\n    return"),
    "swapped_axis": ("__int128 dx = (__int128)px - cx, dy = (__int128)py - cy;\n    return",
                     "__int128 dx = (__int128)px - cy, dy = (__int128)py - cx;\n    return"),
    "knn_reversed_ties": ("return (x->id > y->id) - (x->id < y->id);", "return (x->id < y->id) - (x->id > y->id);"),
    "knn_off_by_one": ("for (int64_t i = 0; i < k; ++i) {\n        out_ids[i] = a[i].id;",
                       "for (int64_t i = 0; i < k; ++i) {\n        out_ids[i] = a[i + (i + 1 < n)].id;"),
}

# polygon x polygon join oracle (oracle/polygon_join_oracle.c) against tests/test_polygon_join_oracle_pins.py
PJ_MUTANTS = {
    "collinear_straddle": ("if (d1 * d2 < 0 && d3 * d4 < 0) return 1;", "if (d1 * d2 <= 0 && d3 * d4 <= 0) return 1;"),
    "no_collinear_touch": ("    return (rx >= (px < qx ? px : qx))", "    return 0 && (rx >= (px < qx ? px : qx))"),
    "one_sided_containment": ("                                                        ring_vertex_inside(&t->A, a, &t->B, b));",
                              "                                                        0);"),
    "first_ring_vertex_only": ("for (int64_t r = Q->pro[q]; r < Q->pro[q + 1]; ++r) {",
                               "for (int64_t r = Q->pro[q]; r < Q->pro[q] + 1 && r < Q->pro[q + 1]; ++r) {"),
    "drop_closing_edge": ("        for (int64_t k = A->ro[r]; k < A->ro[r + 1]; ++k) {",
                          "        for (int64_t k = A->ro[r]; k + 1 < A->ro[r + 1]; ++k) {"),
    "swapped_orient_operand": ("__int128 v = (__int128)(qx - px) * (ry - py) - (__int128)(qy - py) * (rx - px);",
                               "__int128 v = (__int128)(qx - px) * (ry - py) - (__int128)(qy - py) * (rx - qx);"),
}


def _run_mutant(tmp_path, name, src_name, old, new, pins):
    for d in ("oracle", "gen", "tests"):
        shutil.copytree(os.path.join(ROOT, d), tmp_path / d,
                        ignore=shutil.ignore_patterns("liboracle.so", "__pycache__", "*.o"))
    src = tmp_path / "oracle" / src_name
    text = src.read_text()
    assert text.count(old) == 1, f"mutation site for {name} not found"
    src.write_text(text.replace(old, new))
    r = subprocess.run([sys.executable, "-m", "pytest", pins, "-q", "-x",
                        "-p", "no:cacheprovider"], cwd=tmp_path, capture_output=True, text=True, timeout=600)
    assert r.returncode != 0, f"mutant {name} survived the pins:\n{r.stdout[-2000:]}"


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_pins_kill_mutant(name, tmp_path):
    _run_mutant(tmp_path, name, "spade_oracle.c", *MUTANTS[name], "tests/test_oracle_pins.py")


@pytest.mark.parametrize("name", sorted(DIST_MUTANTS))
def test_distance_pins_kill_mutant(name, tmp_path):
    _run_mutant(tmp_path, name, "distance_oracle.c", *DIST_MUTANTS[name], "tests/test_distance_oracle_pins.py")


@pytest.mark.parametrize("name", sorted(PJ_MUTANTS))
def test_polygon_join_pins_kill_mutant(name, tmp_path):
    _run_mutant(tmp_path, name, "polygon_join_oracle.c", *PJ_MUTANTS[name], "tests/test_polygon_join_oracle_pins.py")
