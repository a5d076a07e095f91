"""GPU checks of kernel building blocks (not of the method): the library's
division routine is bitwise IEEE a/b on the operand ranges CloverLeaf uses."""
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    return torch


@pytest.mark.parametrize("emax,seed", [(60, 1), (60, 2), (20, 3), (200, 4), (1023, 5), (1023, 6)])
def test_div_rn_bitwise_equals_ieee_division(cuda, emax, seed):
    from paper_conf_cluster_regulymg15_b200.clover import debug_div_check
    bad, ex = debug_div_check(1 << 31, seed, emax)
    assert bad == 0, f"{bad} mismatches, e.g. {ex[0]!r}/{ex[1]!r}"
