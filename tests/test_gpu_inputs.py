"""The GPU input generator builds the same CSR as the numpy one (bit for bit)."""
import numpy as np
import pytest

from inputs import grid_csr, kronecker_csr, tree4_csr

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gen():
    import inputs.gpu
    inputs.gpu.build()
    return inputs.gpu


@pytest.mark.parametrize("scale,seed", [(6, 1), (10, 1), (14, 3)])
def test_kronecker_twin(gen, scale, seed):
    a = kronecker_csr(scale, 16, seed)
    rp, col = gen.kronecker_csr_cuda(scale, 16, seed)
    assert np.array_equal(rp.cpu().numpy(), a.row_ptr)
    assert np.array_equal(col.cpu().numpy(), a.col)


def test_edge_weight_twin(gen):
    from inputs import edge_weights
    a = kronecker_csr(12, 16, 2)
    rp, col = gen.kronecker_csr_cuda(12, 16, 2)
    w = gen.edge_weights_cuda(rp, col, 7, 255)
    assert np.array_equal(w.cpu().numpy(), edge_weights(a.row_ptr, a.col, 7, 255))


def test_grid_and_tree_twins(gen):
    a = grid_csr(37, 53)
    rp, col = gen.grid_csr_cuda(37, 53)
    assert np.array_equal(rp.cpu().numpy(), a.row_ptr) and np.array_equal(col.cpu().numpy(), a.col)
    a = tree4_csr(10000)
    rp, col = gen.tree4_csr_cuda(10000)
    assert np.array_equal(rp.cpu().numpy(), a.row_ptr) and np.array_equal(col.cpu().numpy(), a.col)
