"""Full-size parity (-m gpu) at BASELINE.json configs[1] sizes, in the launch
configuration bench.py times: the unprotected kernel against the oracle (full
outputs where the oracle is fast, sampled outputs / row bands otherwise), and
every RMT variant bitwise against the unprotected output with zero false
alarms."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads

pytestmark = pytest.mark.gpu

JOBS = None


def _jobs():
    global JOBS
    if JOBS is None:
        JOBS = {j.kernel: j for j in workloads.config_jobs("suite")}
    return JOBS


def _run(j, variant):
    b = j.device_buffers()
    outs = [i for i, h in enumerate(j.host_in) if h is None]
    for i in outs:
        b[i].fill_(-1)
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = rmt.make_workspace(j.kernel, variant, j.n, j.dims)
    rmt.launch(j.kernel, variant, b, j.n, err, dims=j.dims, workspace=ws)
    torch.cuda.synchronize()
    return int(err.item()), [b[i].cpu().numpy().copy() for i in outs]


def _oracle_check(j, outs):
    rng = np.random.default_rng(0)
    if j.kernel == "binarysearch":
        A, q = j.host_in[0], j.host_in[1]
        s = rng.integers(0, q.size, 1 << 14)
        assert np.array_equal(outs[0].view(np.uint32)[s], oracle.binarysearch(A, q[s]))
    elif j.kernel == "fwt":
        assert np.array_equal(outs[0].view(np.uint32), oracle.fwt_f32dag(j.host_in[0]).view(np.uint32))
    elif j.kernel == "prefixsum":
        assert np.array_equal(outs[0].view(np.uint32), oracle.prefixsum_u32(j.host_in[0]))
    elif j.kernel == "reduction":
        assert int(outs[0].view(np.uint64)[0]) == oracle.reduction_u32(j.host_in[0])
    elif j.kernel == "transpose":
        H, W = j.dims
        s = rng.integers(0, H, 256)
        got = outs[0].view(np.uint32).reshape(W, H)
        A = j.host_in[0].reshape(H, W)
        assert np.array_equal(got[:, s], oracle.transpose_u32(A[s]))  # columns of B = rows of A
    elif j.kernel == "sobel":
        H, W = j.dims
        I = j.host_in[0].reshape(H, W).view(np.uint8).reshape(H, W, 4)
        got = outs[0].view(np.uint32).reshape(H, W)
        for r in list(rng.integers(1, H - 1, 48)) + [0, 1, H - 2, H - 1]:
            lo, hi = max(0, r - 1), min(H, r + 2)
            band = oracle.sobel(np.ascontiguousarray(I[lo:hi])).view(np.uint32).reshape(hi - lo, W)
            row = band[r - lo]
            if 0 < r < H - 1:
                assert np.array_equal(got[r], row)
            else:
                assert not got[r].any()  # border rows are 0


@pytest.mark.parametrize("kernel", ["binarysearch", "fwt", "prefixsum", "reduction", "transpose", "sobel"])
def test_fullsize_none_vs_oracle_and_variants_identical(kernel):
    j = _jobs()[kernel]
    err, ref = _run(j, "none")
    assert err == 0
    _oracle_check(j, ref)
    for v in rmt.RMT_VARIANTS:
        for _ in range(2):
            err, outs = _run(j, v)
            assert err == 0, f"{kernel}/{v}: {err} false alarms at full size"
            for a, b in zip(outs, ref):
                assert np.array_equal(a, b), f"{kernel}/{v} differs from none at full size"
