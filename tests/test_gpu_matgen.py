"""The GPU R-MAT generator (matgen/matgen_gpu.cu) is input generation,
not the method; it must reproduce the host generator (matgen.c) exactly -- same keys,
same coalesced CSR, same position-keyed values, same vectors -- so that every oracle
comparison made on host-generated matrices covers the GPU-built ones too."""
import numpy as np
import pytest
import torch

import matgen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("scale,seed", [(8, 3), (12, 61), (15, 62)])
@pytest.mark.parametrize("kind", ["f64", "f32", "int"])
def test_device_rmat_equals_host(scale, seed, kind):
    from matgen import gpu
    A = matgen.rmat(scale, seed=seed, kind=kind)
    dtype = torch.float32 if kind == "f32" else torch.float64
    rp, col, val = gpu.rmat(scale, seed=seed, kind=kind, dtype=dtype)
    assert np.array_equal(rp.cpu().numpy(), A.row_ptr)
    assert np.array_equal(col.cpu().numpy(), A.col)
    assert np.array_equal(val.cpu().double().numpy(), A.val)


def test_device_rmat_value_ranges():
    """values(k0, k1) of any nonzero range equal the full array's slice (rank-local rows)."""
    from matgen import gpu
    g = gpu.DeviceRMAT(13, seed=63)
    full = g.values()
    for k0, k1 in ((0, 1), (5, 5000), (g.nnz - 7, g.nnz), (1234, 99999)):
        assert torch.equal(g.values(k0, k1), full[k0:k1])
        assert torch.equal(g.col(k0, k1), g.col()[k0:k1])


@pytest.mark.parametrize("kind", ["f64", "f32", "int"])
def test_device_vector_equals_host(kind):
    from matgen import gpu
    n = 100003
    ref = matgen.vector(n, 64, 2, kind)
    dtype = torch.float32 if kind == "f32" else torch.float64
    assert np.array_equal(gpu.vector(n, 64, 2, kind, dtype).cpu().double().numpy(), ref)
    assert np.array_equal(gpu.vector(1000, 64, 2, kind, dtype, i0=777).cpu().double().numpy(), ref[777:1777])
