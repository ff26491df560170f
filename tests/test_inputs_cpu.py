"""The seeded input generators (-m "not gpu"): the device twins reproduce the
host streams bit for bit (torch on the CPU device here), and the new input sets
have the structure their tests rely on."""
import numpy as np
import torch

from paper_conf_isca_waddenlgss14_b200 import inputs


def test_device_twins_bitwise():
    for seed, n, off, st in [(1, 1000, 0, 0), (7, 4099, 123456789, 3), (10, 77, (1 << 33) + 5, 22)]:
        a = inputs.u64(seed, n, off, st)
        b = inputs.u64_t(seed, n, off, st, device="cpu").numpy().view(np.uint64)
        assert np.array_equal(a, b)
        assert np.array_equal(inputs.uniform_f32(seed, n, off, st).view(np.uint32),
                              inputs.uniform_f32_t(seed, n, off, st, device="cpu").numpy().view(np.uint32))
    assert np.array_equal(inputs.blackscholes_r(1, 5000, 99).view(np.uint32),
                          inputs.blackscholes_r_t(1, 5000, 99, device="cpu").numpy().view(np.uint32))
    h = inputs.matmul_bf16_normal(10, 64, 96, stream=22).reshape(-1).view(np.int16)
    d = inputs.matmul_bf16_normal_t(10, 64, 96, stream=22, device="cpu").numpy()
    assert np.mean(h == d) > 0.999  # libm vs torch log/cos: a rare last-bit bf16 difference is allowed


def test_new_input_sets():
    prm = inputs.blackscholes_indep(3, 4096)
    S, K, T, R, V = prm
    assert prm.dtype == np.float32 and (S >= 5).all() and (S <= 30).all() and (K >= 1).all() and (K <= 100).all()
    assert (T >= 0.25).all() and (T <= 10).all() and (R >= 0.01).all() and (R <= 0.05).all()
    assert (V >= 0.1).all() and (V <= 0.5).all()
    A, q = inputs.binarysearch_dups(1, 10000, 5000)
    assert (np.diff(A.astype(np.int64)) >= 0).all() and A[0] == 0 and A[-1] == 0xFFFFFFFF
    assert (np.diff(A.astype(np.int64)) == 0).sum() > 5000
    w = inputs.floydwarshall_sparse(1, 64, 0.1)
    assert (np.diag(w) == 0).all() and (w == inputs.FW_INF).mean() > 0.8
    x = inputs.with_specials(inputs.fwt_x(1, 10000), 1, 0.05)
    assert np.isnan(x).any() and (np.signbit(x) & (x == 0)).any() and ((x == 0) & ~np.signbit(x)).any()
    torch.manual_seed(0)
