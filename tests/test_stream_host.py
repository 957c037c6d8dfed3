"""Host logic of the beyond-memory streaming scheduler (mp_plan_stream; no GPU needed)."""
import pytest

from paper_conf_ipps_juryl022_b200 import mstamp

CASES = [  # (d, n, m, prec, exclusion, self_join)
    (64, 262144, 256, "fp32", 64, True),      # C3
    (128, 1 << 20, 256, "fp32", -1, False),   # C4
    (256, 1 << 21, 512, "fp64", 128, True),   # C5
    (256, 1 << 21, 512, "mixed", 128, True),
    (16, 65536, 128, "fp16", 32, True),
]


@pytest.mark.parametrize("case", CASES)
def test_plan_stream_monotone_and_aligned(case):
    """Rows per chunk and diagonals per band grow with the budget, never exceed the (tile-height
    rounded) problem, and the band is about twice the row window."""
    d, n, m, prec, e, self_join = case
    prev = (0, 0)
    for budget in [2 << 30, 4 << 30, 16 << 30, 64 << 30, 512 << 30]:
        try:
            R, Wb = mstamp.plan_stream(d, n, m, prec, e, self_join, budget)
        except mstamp.MPError as ex:
            assert ex.status == 2 and prev == (0, 0)   # NOMEM only below the smallest workable budget
            continue
        assert R >= prev[0] and Wb >= prev[1]
        assert R > 0 and Wb >= R and R % 64 == 0
        assert R <= n + 4096
        prev = (R, Wb)
    assert prev[0] > 0


def test_plan_stream_whole_problem_with_a_large_budget():
    R, Wb = mstamp.plan_stream(4, 4096, 64, "fp64", 16, True, 64 << 30)
    assert R >= 4096


def test_plan_stream_rejects_tiny_budget_and_bad_args():
    with pytest.raises(mstamp.MPError) as ei:
        mstamp.plan_stream(64, 262144, 256, "fp32", 64, True, 1 << 20)
    assert ei.value.status == 2
    with pytest.raises(mstamp.MPError) as ei:
        mstamp.plan_stream(64, 262144, 256, "fp32", 64, True, 0)
    assert ei.value.status == 1
    with pytest.raises(mstamp.MPError):
        mstamp.plan_stream(64, 262144, 256, 9, 64, True, 1 << 30)


def test_plan_stream_rows_scale_with_budget():
    """Doubling the budget (well above the fixed granule margins) about doubles the row window."""
    R1, _ = mstamp.plan_stream(64, 1 << 22, 256, "fp32", 64, True, 8 << 30)
    R2, _ = mstamp.plan_stream(64, 1 << 22, 256, "fp32", 64, True, 16 << 30)
    assert 1.8 <= R2 / R1 <= 2.2
