"""The GPU generator (graphgen/gpu.py) reproduces the CPU generator bit for bit."""
import numpy as np
import pytest

import graphgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ggpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import graphgen.gpu as gg
    return gg


def same(cpu, dev):
    assert dev.n == cpu.n and dev.m == cpu.m
    np.testing.assert_array_equal(dev.offsets.cpu().numpy(), cpu.offsets)
    np.testing.assert_array_equal(dev.col.cpu().numpy(), cpu.col)
    np.testing.assert_array_equal(dev.w.cpu().numpy().view(np.uint32), cpu.w.view(np.uint32))


@pytest.mark.parametrize("scale,ef,seed,weights", [(10, 16, 1, "uniform"), (14, 16, 3, "paper"),
                                                   (16, 8, 2, "uniform"), (12, 16, 5, "ones")])
def test_rmat_identical(ggpu, scale, ef, seed, weights):
    same(graphgen.rmat(scale, ef, seed=seed, weights=weights),
         ggpu.rmat(scale, ef, seed=seed, weights=weights))


def test_rmat_many_buckets(ggpu):
    # force many source-range buckets
    same(graphgen.rmat(13, 16, seed=4), ggpu.rmat(13, 16, seed=4, bucket_entries=1 << 12))


def test_rmat_host_output(ggpu):
    """host_out: bucket-by-bucket assembly in pinned host memory gives the same CSR."""
    hg = ggpu.rmat(13, 16, seed=4, bucket_entries=1 << 12, host_out=True)
    assert hg.offsets.device.type == "cpu" and hg.offsets.is_pinned()
    same(graphgen.rmat(13, 16, seed=4), hg)


@pytest.mark.parametrize("n,d", [(1000, 6.0), (1 << 15, 16.0), (12345, 3.5)])
def test_er_identical(ggpu, n, d):
    same(graphgen.er(n, d, seed=7), ggpu.er(n, d, seed=7))


@pytest.mark.parametrize("side,keep,weights", [(64, 1.0, "uniform"), (100, 0.6, "paper"),
                                               (128, 1.0, "gradient"), (33, 0.6, "ones")])
def test_mesh_identical(ggpu, side, keep, weights):
    same(graphgen.mesh(side, keep=keep, seed=2, weights=weights),
         ggpu.mesh(side, keep=keep, seed=2, weights=weights))
