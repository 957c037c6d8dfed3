"""bench.py host logic on CPU: the roofline accounting and the reference arm's JSON line.

The accounting is pinned to things other than itself: the comparator count of Batcher's
odd-even merge sort on N = 2^p inputs has the closed form (p^2 - p + 4) 2^(p-2) - 1 (Knuth,
TAOCP vol. 3, 5.3.4), the computed-cell count of the self-join triangle is a brute-force count
of the cells j - i > e, and the reference arm runs the oracle on a tiny sample and must print
one contract-conforming line.
"""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


@pytest.mark.parametrize("N,ce", [(1, 0), (2, 1), (4, 5), (8, 19), (16, 63), (32, 191), (64, 543),
                                  (128, 1471), (256, 3839)])
def test_batcher_comparator_counts(N, ce):
    # odd-even merge sort of 2^p inputs: (p^2 - p + 4) 2^(p-2) - 1 comparators
    assert bench.batcher_ce(N) == ce
    if N >= 2:
        p = N.bit_length() - 1
        assert ce == (p * p - p + 4) * 2 ** (p - 2) - 1


@pytest.mark.parametrize("cfg,ops", [("C1", 9.5), ("C2", 14.9), ("C3", 24), ("C4", 27), ("C5", 37)])
def test_alu_ops_model_matches_survey(cfg, ops):
    """The roofline's op count per computed cell*dim reproduces SURVEY.md 8(d)'s table (clamp 1 +
    2 CE(d_pad)/d + 3 per profile side), written from the paper's algorithm before any kernel:
    9.5 / 14.9 / 24 / 27 / 37 for C1..C5."""
    from paper_conf_ipps_juryl022_b200 import datagen
    join, d, n, m, e, seed = datagen.CONFIGS[cfg]
    assert bench.alu_ops_per_cell_dim(d, join == "self") == pytest.approx(ops, abs=0.06)


def test_alu_ops_half_modes_count_pairs():
    # half2 instructions serve two cells
    assert bench.alu_ops_mode(16, True, "mixed") == pytest.approx(bench.alu_ops_per_cell_dim(16, True) / 2)
    assert bench.alu_ops_filtered(16, True) < bench.alu_ops_per_cell_dim(16, True)


@pytest.mark.parametrize("n,e", [(10, 0), (10, 2), (37, 5), (8, 7), (8, 9)])
def test_computed_cells_bruteforce(n, e):
    brute = sum(1 for i in range(n) for j in range(i + 1, n) if j - i > e)
    assert bench.computed_cells(n, e, True) == brute
    assert bench.computed_cells(n, e, False) == n * n


def test_reference_arm_json_line():
    """`bench.py --impl reference` (the oracle on host cores) prints one JSON line with the
    contract's keys; no GPU is touched."""
    import oracle
    oracle.build()
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--config", "C1", "--steps", "1", "--warmup", "1", "--ref-seconds", "0.5"],
                         capture_output=True, text=True, env=env, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.strip().startswith("{")]
    assert len(lines) == 1
    j = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in j, k
    assert j["impl"] == "reference" and j["value"] > 0 and j["cpu_baseline"]["kind"] == "oracle"
    assert j["e2e"]["h2d_bytes_per_step"] == 0 and j["e2e"]["value"] == j["value"]
