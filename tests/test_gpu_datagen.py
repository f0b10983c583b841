"""Generator pin (SURVEY §8(c) "Generator pins"): the seeded input generators run on the GPU for the
full-size workloads and on the CPU for the oracle's inputs, so the two must be bit-identical for the
same seed -- every workload kind, both sides, n up to 2^24 (integer-only sampling: splitmix64 draws
searched in 63-bit fixed-point interval arrays, a seeded rank -> key bijection)."""
import pytest
import torch

import datagen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kind,n,theta", [("zipf", 1 << 24, 1.0), ("zipf", (1 << 20) + 3, 0.5), ("zipf", 1 << 18, 1.5),
                                          ("uniform", 1 << 20, 0.0), ("pkfk", (1 << 22) + 1, 0.0),
                                          ("pkfk_zipf", 1 << 20, 1.0), ("graph", 1 << 22, 0.909)])
def test_generators_bit_identical_cpu_cuda(kind, n, theta):
    cpu = datagen.make_workload(kind, n, theta, seed=0x6A5, device="cpu")
    gpu = datagen.make_workload(kind, n, theta, seed=0x6A5, device="cuda")
    for c, g in zip(cpu, gpu):
        assert c.dtype == g.dtype and c.shape == g.shape
        assert torch.equal(c, g.cpu())
