"""GPU parity (-m gpu): CUDA path vs oracle, RMT variants vs the unprotected
kernel (bitwise), determinism, and single-bit fault detection, all through the
C ABI (librmt.so)."""
import numpy as np
import pytest
import torch

from paper_conf_isca_waddenlgss14_b200 import rmt
from cases import DCT, Case, PrefixSum, small_cases
from helpers import VARIANTS, run

pytestmark = pytest.mark.gpu

CASES = small_cases()
IDS = [c.id for c in CASES]


def _run_case(case, variant):
    b = case.buffers()
    err = run(case.kernel, variant, b, case.n, case.dims)
    return err, case.outputs(b)


@pytest.mark.parametrize("case", CASES, ids=IDS)
def test_none_matches_oracle(case):
    err, outs = _run_case(case, "none")
    assert err == 0
    case.check(outs)


@pytest.mark.parametrize("variant", rmt.RMT_VARIANTS)
@pytest.mark.parametrize("case", CASES, ids=IDS)
def test_variant_bit_identical_to_none(case, variant):
    _, ref = _run_case(case, "none")
    for _ in range(2):  # determinism: two runs
        err, outs = _run_case(case, variant)
        assert err == 0, f"{variant}: {err} false alarms"
        for a, b in zip(outs, ref):
            assert np.array_equal(a, b), f"{variant} output differs from none"


FAULT_CASES = [c for c in CASES if c.n >= 1000]


@pytest.mark.parametrize("variant", rmt.RMT_VARIANTS)
@pytest.mark.parametrize("replica", [0, 1])
@pytest.mark.parametrize("case", FAULT_CASES, ids=[c.id for c in FAULT_CASES])
def test_store_value_fault_detected(case, replica, variant):
    """A flipped store value in one replica: exactly one mismatching commit, the
    faulted word is not committed (sentinel kept), everything else is clean."""
    _, ref = _run_case(case, "none")
    rng = np.random.default_rng(case.n + replica)
    fe, e = case.fault_target(rng)
    bit = int(rng.integers(0, 32))
    rmt.inject_fault(replica, "store_val", bit, fe)
    try:
        err, outs = _run_case(case, variant)
    finally:
        rmt.clear_faults()
    assert err == 1
    if case.kernel == "reduction":
        return  # the uncommitted word is a per-CTA partial in the workspace
    o = outs[0].reshape(-1)
    r = ref[0].reshape(-1)
    # dup_kernel compares the two shadow outputs in aligned 4-word groups,
    # whatever the kernel's own store pattern
    grp = Case.commit_group(case, e) if variant == "dup_kernel" else case.commit_group(e)
    if case.fault_propagates():
        # in-place iterative kernel: the suppressed store feeds later passes
        assert not np.array_equal(o[grp], r[grp]), "faulted commit must not be stored"
        return
    if getattr(case, "multipass", False):
        # in-place multi-pass kernel: the suppressed final store leaves the
        # previous pass's intermediate in place (not the committed result)
        assert not np.array_equal(o[grp], r[grp]), "faulted commit must not be stored"
    else:
        assert np.all(o[grp] == 0xFFFFFFFF), "faulted commit must not be stored"
    mask = np.ones(o.size, bool)
    mask[grp] = False
    assert np.array_equal(o[mask], r[mask])
    for a, b in zip(outs[1:], ref[1:]):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("case", FAULT_CASES, ids=[c.id for c in FAULT_CASES])
def test_fault_is_live_in_none(case):
    """Liveness control: the same flip in the unprotected kernel corrupts the output."""
    _, ref = _run_case(case, "none")
    fe, e = case.fault_target(np.random.default_rng(1))
    rmt.inject_fault(0, "store_val", 5, fe)
    try:
        err, outs = _run_case(case, "none")
    finally:
        rmt.clear_faults()
    assert err == 0
    assert any(not np.array_equal(a, b) for a, b in zip(outs, ref))


@pytest.mark.parametrize("variant", sorted(set(["none", *rmt.RMT_VARIANTS])))
def test_prefixsum_carry_in(variant):
    """The multi-GPU shard offset (dims[0] = carry-in) is added to every output."""
    import oracle
    from cases import PrefixSum
    c = PrefixSum(4096 * 5 + 7)
    carry = 0xFFFFFF00
    b = c.buffers()
    err = run("prefixsum", variant, b, c.n, dims=(carry,))
    assert err == 0
    y = c.outputs(b)[0].astype(np.uint64)
    ref = (oracle.prefixsum_u32(c.x).astype(np.uint64) + carry) % 2**32
    assert np.array_equal(y, ref)


def test_cluster_placement_probe():
    """inter_cluster SoR: how often do the two CTAs of a pair share an SM?"""
    pairs = 4096
    same = rmt.probe_cluster_placement(pairs)
    assert 0 <= same <= pairs
    print(f"cluster pairs sharing an SM: {same}/{pairs}")


@pytest.mark.parametrize("variant", sorted(set(["none", *rmt.RMT_VARIANTS])))
@pytest.mark.parametrize("make", [lambda: PrefixSum(4096 * 9 + 5), lambda: DCT(32, 264)], ids=["prefixsum", "dct"])
def test_input_only_16byte_aligned(make, variant):
    """DCT and PrefixSum take 256-bit loads when the input is 32-B aligned and
    16-B loads otherwise (the ABI minimum is 16 B): an input placed 16 B past a
    32-B boundary must give the same bits, against the oracle."""
    from helpers import dev

    case = make()
    b = case.buffers()
    src = b[0].reshape(-1)
    pad = torch.empty(src.numel() + 8, dtype=src.dtype, device="cuda")
    assert pad.data_ptr() % 32 == 0
    shifted = pad[4: 4 + src.numel()]
    assert shifted.data_ptr() % 32 == 16
    shifted.copy_(src)
    b[0] = shifted.view(b[0].shape)
    err = run(case.kernel, variant, b, case.n, case.dims)
    assert err == 0
    case.check(case.outputs(b))


def test_pipelined_host_path_matches_oracle():
    """rmt_run_host_variants_pipelined (bench.py's e2e leg): several kernels in a
    row, inputs / launches / outputs on three streams, no host sync until the
    end -- every output equals the oracle and every error count is 0."""
    import oracle
    from cases import BinarySearch, FloydWarshall, PrefixSum
    variants = ["none", "intra_reg", "inter_group", "inter_cluster"]
    cases = [BinarySearch(70001, 5003), PrefixSum(4096 * 7 + 3), FloydWarshall(64)]
    streams = (torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream())
    runs = []
    for c in cases:
        dev = c.buffers()
        host = [t.cpu().pin_memory() for t in dev]
        errd = torch.zeros(len(variants), dtype=torch.int64, device="cuda")
        errh = torch.zeros(len(variants), dtype=torch.int64).pin_memory()
        wsl = [rmt.make_workspace(c.kernel, v, c.n, c.dims) for v in variants]
        torch.cuda.synchronize()
        rmt.run_host_variants_pipelined(c.kernel, variants, host, dev, c.n, errd, wsl, errh, streams, dims=c.dims)
        runs.append((c, host, errh, dev, wsl))
    for s in streams:
        s.synchronize()
    for c, host, errh, dev, wsl in runs:
        assert errh.tolist() == [0] * len(variants), f"{c.kernel}: {errh.tolist()}"
        if c.kernel == "floydwarshall":  # D in/out (the last variant's result), P out
            c.check([host[0].numpy().view(np.uint32).reshape(c.n, c.n), host[1].numpy().view(np.uint32).reshape(c.n, c.n)])
        else:
            c.check([host[-1].numpy().view(np.uint32).reshape(-1)])
