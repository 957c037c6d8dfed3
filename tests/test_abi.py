"""C-ABI library: loads without a GPU, exports every symbol include/mp.h declares, and the
host-side scheduler (diagonal-band plan) is correct.  No compute calls (CPU only)."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_juryl022_b200 import build, mstamp
    build.build()
    return mstamp.load()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "mp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mp_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(lib):
    syms = declared_symbols()
    assert len(syms) >= 10
    for s in syms:
        assert hasattr(lib, s), s
    from paper_conf_ipps_juryl022_b200 import mstamp
    assert sorted(mstamp.EXPORTS) == syms


def test_version(lib):
    from paper_conf_ipps_juryl022_b200 import mstamp
    assert "sm_100a" in mstamp.version()


def test_key_words(lib):
    from paper_conf_ipps_juryl022_b200 import mstamp
    assert mstamp.key_words(16, 100, "fp32") == 1600
    assert mstamp.key_words(16, 100, "fp64") == 3200


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("cfg", [(16, 65536, 128, 32, True), (128, 1 << 20, 256, 0, False),
                                 (256, 1 << 21, 512, 128, True), (4, 4096, 64, 16, True), (3, 50, 8, 2, True)])
def test_band_plan(lib, cfg, world):
    """Equal-cell diagonal bands: contiguous, cover all cells, balanced to a block."""
    from paper_conf_ipps_juryl022_b200 import mstamp
    d, n, m, e, self_join = cfg
    bb, cells = mstamp.plan_bands(d, n, m, "fp32", e, self_join, world)
    assert bb[0] == 0 and np.all(np.diff(bb) >= 0)
    total = (n - e - 1) * (n - e) // 2 if self_join else n * n
    assert cells.sum() == total
    block_max = 64 * n   # a diagonal block holds at most 64 diagonals
    assert cells.max() - cells.min() <= 2 * block_max


def test_init_without_gpu_fails_cleanly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_ipps_juryl022_b200 import mstamp
    with pytest.raises(mstamp.MPError):
        mstamp.Context(0)


def test_invalid_plan_args(lib):
    from paper_conf_ipps_juryl022_b200 import mstamp
    with pytest.raises(mstamp.MPError):
        mstamp.plan_bands(0, 100, 8)
    with pytest.raises(mstamp.MPError):
        mstamp.plan_bands(4, 100, 1)


def test_product_path_does_not_touch_oracle():
    """The CUDA path never imports / links the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_juryl022_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "oracle_" not in txt and "liboracle" not in txt, f
