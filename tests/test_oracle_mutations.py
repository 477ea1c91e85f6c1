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


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_pins_kill_mutant(name, tmp_path):
    old, new = MUTANTS[name]
    for d in ("oracle", "gen", "tests"):
        shutil.copytree(os.path.join(ROOT, d), tmp_path / d,
                        ignore=shutil.ignore_patterns("liboracle.so", "__pycache__", "*.o"))
    src = tmp_path / "oracle" / "spade_oracle.c"
    text = src.read_text()
    assert text.count(old) == 1, f"mutation site for {name} not found"
    src.write_text(text.replace(old, new))
    r = subprocess.run([sys.executable, "-m", "pytest", "tests/test_oracle_pins.py", "-q", "-x",
                        "-p", "no:cacheprovider"], cwd=tmp_path, capture_output=True, text=True, timeout=600)
    assert r.returncode != 0, f"mutant {name} survived the pins:\n{r.stdout[-2000:]}"
