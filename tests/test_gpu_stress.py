"""Inter-group queue protocol under stress (-m gpu; SURVEY 8(c) "C-Q
inter-group ring" pins, PAPER.md P:691 two-tier locking, P:693 coherent reads).

Every kernel runs under inter_group (L2 queue) and inter_cluster (DSMEM
mailbox) in the STRESS instantiation (rmt_set_stress, include/rmt.h): ring depth
1, 2 or 8 (depth 1 forces a hand-over per record and exercises the
free-before-wait rule on both sides), random per-CTA and per-commit
__nanosleep skew, and a (pair, warp, sequence) tag folded into every record key
(a record consumed out of order, twice or from another ring is counted as a
mismatch).  Grids are tens to hundreds of times the resident capacity, so
queue regions are handed from pair to pair many times.  Every run must be
bitwise equal to the unprotected output with err == 0, and leave the queue's
control block zeroed (ticket, done, watchdog flag: the self-reset ran, so all
2C tickets were taken).  A dropped producer must end in the watchdog: err >= 1,
the sticky flag reported by rmt_workspace_status, and the same workspace clean
and correct on the next launch.
"""
import numpy as np
import pytest
import torch

from paper_conf_isca_waddenlgss14_b200 import rmt
from cases import (DCT, DWT, FWT, BinomialOption, BitonicSort, BinarySearch, BlackScholes, FloydWarshall, MatMul,
                   PrefixSum, Reduction, Sobel, Transpose)

pytestmark = pytest.mark.gpu

STRESS_CASES = [
    lambda: BlackScholes(1 << 24),
    lambda: BinarySearch(1 << 20, 1 << 22),
    lambda: FWT(1 << 22),
    lambda: PrefixSum(1 << 24),
    lambda: Reduction(1 << 24),
    lambda: Transpose(2048, 4096),
    lambda: Sobel(2048, 2048),
    lambda: FloydWarshall(128),
    lambda: DCT(1024, 2048),
    lambda: MatMul(512, 512, 256, integer=True),
    lambda: DWT(1 << 22),
    lambda: BitonicSort(1 << 18),
    lambda: BinomialOption(1 << 13),
]
_cache = {}


def _case(i):
    if i not in _cache:
        c = STRESS_CASES[i]()
        b = c.buffers()
        err = _launch(c, "none", b)
        assert err == 0
        _cache[i] = (c, c.outputs(b))
    return _cache[i]


def _launch(case, variant, bufs, ws=None):
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    if ws is None:
        ws = rmt.make_workspace(case.kernel, variant, case.n, case.dims)
    rmt.launch(case.kernel, variant, bufs, case.n, err, dims=case.dims, workspace=ws)
    torch.cuda.synchronize()
    return int(err.item())


@pytest.fixture(autouse=True)
def _reset_stress():
    yield
    rmt.set_stress(0, 0, 0, 0)


@pytest.mark.parametrize("depth", [1, 2, 8])
@pytest.mark.parametrize("variant", ["inter_group", "inter_cluster"])
@pytest.mark.parametrize("idx", range(len(STRESS_CASES)), ids=[f().kernel for f in STRESS_CASES])
def test_queue_stress(idx, variant, depth):
    case, ref = _case(idx)
    ws = rmt.make_workspace(case.kernel, variant, case.n, case.dims)
    rmt.set_stress(depth, rmt.STRESS_TAGS | rmt.STRESS_SKEW, 400, 0)
    for rep in range(2):
        b = case.buffers()
        err = _launch(case, variant, b, ws)
        assert err == 0, f"{case.kernel}/{variant} depth {depth}: {err} mismatches (tags/order/values)"
        for a, r in zip(case.outputs(b), ref):
            assert np.array_equal(a, r), f"{case.kernel}/{variant} depth {depth} differs from none"
        if variant == "inter_group":
            ctrl = ws[:12].view(torch.int32).cpu().numpy()
            assert ctrl[0] == 0 and ctrl[1] == 0 and ctrl[2] == 0, f"control block not reset: {ctrl}"
            assert rmt.workspace_status(variant, ws) is None


@pytest.mark.parametrize("variant", ["inter_group", "inter_cluster"])
def test_dropped_producer_hits_watchdog(variant):
    case = BlackScholes(1 << 18)
    b = case.buffers()
    assert _launch(case, "none", b) == 0
    ref = case.outputs(b)
    ws = rmt.make_workspace(case.kernel, variant, case.n, case.dims)
    rmt.set_stress(8, rmt.STRESS_DROP, 0, 1 << 20)  # ~0.5 ms watchdog
    b = case.buffers()
    err = _launch(case, variant, b, ws)
    assert err >= 1, "a lost producer must be reported"
    # pair 0's stores were never committed (sentinel); every other pair is intact
    lost = case.outputs(b)
    assert np.all(lost[0][:1024] == 0xFFFFFFFF)
    assert np.array_equal(lost[0][1024:], ref[0][1024:])
    if variant == "inter_group":
        msg = rmt.workspace_status(variant, ws)
        assert msg is not None and "watchdog" in msg
        assert rmt.workspace_status(variant, ws) is None  # cleared
    rmt.set_stress(0, 0, 0, 0)
    b = case.buffers()
    assert _launch(case, variant, b, ws) == 0  # the workspace is reusable
    for a, r in zip(case.outputs(b), ref):
        assert np.array_equal(a, r)
