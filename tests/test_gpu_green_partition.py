"""The multi-GPU (8xB200) code path on one GPU: every x-slab's stream lives on
its own SM-disjoint green context (CUDA driver API, tools/green_partition.py),
so a slab's spinning protocol CTAs and its PDL-parked CTAs never hold the SMs
its neighbour needs -- as on separate GPUs.  With LBMR_TEST_OTHER_GPU=1 the
library treats the neighbours as ranks on other GPUs: in-kernel halo waits in
the level and gather kernels, no wait kernels, the PDL chain on (the
configuration the driver's 8-GPU runs use).  The slabs must
equal one grid bitwise."""
import os
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _green():
    sys.path.insert(0, ROOT)
    try:
        from cuda.bindings import driver as d  # noqa: F401
    except ImportError:
        pytest.skip("cuda-python driver bindings not available")
    from tools import green_partition
    return green_partition


@pytest.mark.parametrize("P,steps,name", [(2, 6, "tunnel4_s5"), (4, 6, "tunnel4_s5"), (8, 6, "tunnel4_s5"),
                                          (2, 8, "cavity2"), (3, 4, "kbc_mini")])
def test_green_partition_equals_single_grid(P, steps, name, monkeypatch):
    monkeypatch.setenv("LBMR_TEST_OTHER_GPU", "1")
    gp = _green()
    assert gp.run(P, steps, name) == 0.0


def test_green_partition_repeated(monkeypatch):
    """Eight slabs, five fresh runs: no run differs (a protocol race would
    show as a rare mismatch or a timed-out wait)."""
    monkeypatch.setenv("LBMR_TEST_OTHER_GPU", "1")
    gp = _green()
    for _ in range(5):
        assert gp.run(8, 4, "tunnel4_s5") == 0.0
