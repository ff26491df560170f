"""Fault-injection campaign (-m gpu): single-bit flips at every instrumented
site of every kernel, in either replica, under every RMT variant.

For each (kernel, site, element, bit) the same flip is first injected into the
unprotected kernel: the fault is *live* iff it changes the output (faults
masked by the computation are not silent data corruption).  Every live fault
inside the sphere of replication must then be detected (err >= 1) by every RMT
variant, in either replica; STORE_* flips corrupt exactly one commit, so they
must give err == 1 exactly.  Sites outside the SoR by design are not expected
to be caught; for intra_nolds (-LDS) the kernel's
shared memory is such a site, and an SMEM flip must stay silent.
"""
import numpy as np
import pytest

from paper_conf_isca_waddenlgss14_b200 import rmt
from cases import (DCT, DWT, FWT, BinomialOption, BitonicSort, BinarySearch, BlackScholes, FloydWarshall, MatMul, PrefixSum, Reduction, Sobel,
                   Transpose)
from helpers import run

pytestmark = pytest.mark.gpu

# kernel case, sites with their element-index space (callable(case) -> upper bound)
CAMPAIGN = [
    (lambda: BlackScholes(5000), {"load": lambda c: c.n, "compute": lambda c: c.n, "store_val": lambda c: c.n,
                                  "store_addr": lambda c: c.n}),
    # BinarySearch SMEM = an entry of the shared-memory table L_1 = A[32 j] (2048
    # entries at N = 2^16), flipped where the binary search reads it
    (lambda: BinarySearch(1 << 16, 4000), {"load": lambda c: c.Q, "compute": lambda c: c.Q,
                                           "smem": lambda c: (c.N + 31) // 32,
                                           "store_val": lambda c: c.Q, "store_addr": lambda c: c.Q}),
    (lambda: FWT(1 << 14), {"load": lambda c: c.n, "compute": lambda c: c.n, "smem": lambda c: c.n,
                            "store_val": lambda c: c.n, "store_addr": lambda c: c.n}),
    # PrefixSum SMEM = warp total i of chunk ch (element ch*256 + i): the unprotected
    # scan reads 32 (sub-tile, warp) totals per chunk, the intra variants 16 (warp)
    # totals, so i < 16 is a site every variant has; the intra layout's last total
    # (i = 15) feeds no later warp of the tile (dead there, live in none), so the
    # sampled sites are i < 15, live in every layout
    (lambda: PrefixSum(4096 * 9 + 5), {"load": lambda c: c.n, "compute": lambda c: 256 * 10,
                                       "smem": lambda c: (lambda rng: 256 * int(rng.integers(0, 10)) +
                                                          int(rng.integers(0, 15))),
                                       "store_val": lambda c: c.n, "store_addr": lambda c: c.n}),
    (lambda: Reduction(300007), {"load": lambda c: c.n, "compute": lambda c: 1184 * 256,
                                 "smem": lambda c: 1184 * 8, "store_val": lambda c: 1, "store_addr": lambda c: 1}),
    (lambda: Transpose(96, 160), {"load": lambda c: c.n, "smem": lambda c: c.n, "store_val": lambda c: c.n,
                                  "store_addr": lambda c: c.n}),
    (lambda: Sobel(72, 132), {"load": lambda c: c.n, "compute": lambda c: c.n, "store_val": lambda c: c.n,
                              "store_addr": lambda c: c.n}),
    (lambda: DCT(32, 264), {"load": lambda c: c.n, "compute": lambda c: c.n, "smem": lambda c: c.n,
                            "store_val": lambda c: c.n, "store_addr": lambda c: c.n}),
    (lambda: FloydWarshall(48), {"load": lambda c: c.n ** 3, "compute": lambda c: c.n ** 3,
                                 "store_val": lambda c: c.n ** 3, "store_addr": lambda c: c.n ** 3}),
    # MatMul LOAD = an A operand word after TMA, SMEM = a Bt operand word (both in the
    # shared-memory stage the tensor core reads); K = 2048 spans two TMEM chunks
    (lambda: MatMul(256, 256, 2048), {"load": lambda c: c.M * c.K, "smem": lambda c: c.N * c.K,
                                      "compute": lambda c: c.n, "store_val": lambda c: c.n,
                                      "store_addr": lambda c: c.n}),
    (lambda: BitonicSort(1 << 14), {"load": lambda c: c.n, "compute": lambda c: c.n, "smem": lambda c: c.n,
                                    "store_val": lambda c: c.n, "store_addr": lambda c: c.n}),
    (lambda: BinomialOption(2000), {"load": lambda c: c.n, "compute": lambda c: c.n, "store_val": lambda c: c.n,
                                    "store_addr": lambda c: c.n}),
    (lambda: DWT(1 << 14), {"load": lambda c: c.n, "compute": lambda c: c.n // 2, "smem": lambda c: c.n // 2,
                            "store_val": lambda c: c.n, "store_addr": lambda c: c.n}),
]
SAMPLES = 24  # live faults per (kernel, site)


def _silent_by_design(kernel, variant, site):
    """Sites outside a variant's sphere of replication:
    -LDS shares the kernel's shared memory (Table 2 "LDS x" for -LDS);
    MatMul's single-copy intra variants share the operand tiles the tensor core
    reads (the load path is outside the SoR; +LDS duplicates them)."""
    if variant == "intra_nolds" and site == "smem":
        return True
    return kernel == "matmul" and variant in ("intra_reg", "intra_nolds") and site in ("load", "smem")


def _outputs(case, variant):
    b = case.buffers()
    err = run(case.kernel, variant, b, case.n, case.dims)
    return err, case.outputs(b)


def _with_fault(case, variant, replica, site, bit, elem):
    rmt.inject_fault(replica, site, bit, elem)
    try:
        return _outputs(case, variant)
    finally:
        rmt.clear_faults()


@pytest.mark.parametrize("idx", range(len(CAMPAIGN)), ids=[f().kernel for f, _ in CAMPAIGN])
def test_fault_campaign(idx):
    make, sites = CAMPAIGN[idx]
    case = make()
    _, ref = _outputs(case, "none")
    rng = np.random.default_rng(1000 + idx)
    report = {}
    for site, bound in sites.items():
        live = detected = predicted = 0
        for _ in range(SAMPLES * (40 if case.kernel == "floydwarshall" else 4)):
            if live >= SAMPLES:
                break
            b = bound(case)
            elem = int(b(rng)) if callable(b) else int(rng.integers(0, b))
            bit = int(rng.integers(0, 32))
            if site == "store_addr":
                pass  # any of the 32 index bits: out-of-range or misaligned flips are dropped by none (liveness)
            _, o0 = _with_fault(case, "none", 0, site, bit, elem)
            pred = case.flipped_oracle(elem, bit) if site == "load" else None
            if pred is not None:
                # LOAD liveness predicted by the oracle on the flipped input word
                # (independent of the kernel): the unprotected kernel's faulted
                # output must be exactly that
                for a, b in zip(o0, pred):
                    assert np.array_equal(np.asarray(a).reshape(-1), np.asarray(b).reshape(-1)), \
                        f"{case.kernel}: none with a flipped input word != oracle on the flipped input"
                predicted += 1
            if all(np.array_equal(a, b) for a, b in zip(o0, ref)):
                continue  # masked by the computation: not an SDC, nothing to detect
            live += 1
            for variant in rmt.RMT_VARIANTS:
                for replica in (0, 1):
                    err, _ = _with_fault(case, variant, replica, site, bit, elem)
                    if _silent_by_design(case.kernel, variant, site):
                        # both replicas read the one flipped copy -> no mismatch, silent
                        assert err == 0, f"{case.kernel}/{variant}: {site} fault should be silent (err {err})"
                        continue
                    assert err >= 1, (f"{case.kernel}: live {site} fault (elem {elem}, bit {bit}) in replica "
                                      f"{replica} NOT detected by {variant}")
                    if variant == "dup_kernel" and site == "store_addr":
                        # output comparison sees an address flip as two differing groups (the
                        # skipped one, left poisoned, and the overwritten one), not as one commit
                        assert err <= 2 or case.kernel == "floydwarshall"
                    elif site.startswith("store") and case.kernel not in ("floydwarshall",):
                        assert err == 1, f"{case.kernel}/{variant}: {site} flip must corrupt exactly one commit"
                    detected += 1
        report[site] = (live, detected, predicted)
        assert live > 0, f"{case.kernel}/{site}: no live fault found (vacuous)"
    print(case.kernel, report)
