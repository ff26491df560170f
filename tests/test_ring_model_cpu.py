"""CPU model of the inter-group queue protocol (-m "not gpu"; SURVEY 8(c)
"C-Q inter-group ring": a std::atomic model of the same protocol under stress).

tests/model/ring_model.cpp restates the protocol of rmt_device.cuh (V_INTER)
with C++ atomics, one thread per CTA role and a pool of worker threads standing
in for the resident CTA slots: region turns (first tier) and per-slot 64-bit
records (marker j + 1, digest) freed by the consumer (second tier).  Every
configuration must finish (no deadlock) with every record consumed once, in
order, with its producer's (pair, sequence) digest, and leave the control block
and every slot zeroed -- at ring depth 1, 2, 4 and 8, one region (every pair
hands the ring to the next) or several, and down to 2 workers (the minimum
residency the deadlock-freedom argument needs).  Mutants that drop the
consumer's free or the producer's wait for a free slot must fail, so the model
can tell the difference.
"""
import os
import subprocess

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "model", "ring_model.cpp")


def _build(tmp_path, src_text=None, name="ring_model"):
    src = SRC
    if src_text is not None:
        src = str(tmp_path / f"{name}.cpp")
        with open(src, "w") as f:
            f.write(src_text)
    exe = str(tmp_path / name)
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-pthread", "-o", exe, src])
    return exe


@pytest.fixture(scope="module")
def model(tmp_path_factory):
    return _build(tmp_path_factory.mktemp("ring"))


@pytest.mark.parametrize("S", [1, 2, 4, 8])
@pytest.mark.parametrize("R,workers", [(1, 2), (2, 3), (4, 8), (64, 16)])
def test_ring_protocol_model(model, S, R, workers):
    for seed in range(3):
        r = subprocess.run([model, str(S), str(R), str(workers), "48", "60", str(seed + 17 * S + R), "3"],
                           capture_output=True, text=True, timeout=60)
        assert r.returncode == 0, r.stderr[-2000:]
        assert r.stdout.startswith("ok")


def _mutant_fails(tmp_path, old, new, name):
    text = open(SRC).read()
    assert old in text
    exe = _build(tmp_path, text.replace(old, new), name)
    failures = 0
    for seed in range(1, 4):
        try:
            r = subprocess.run([exe, "2", "1", "2", "16", "40", str(seed), "2"], capture_output=True, text=True,
                               timeout=10)
            failures += r.returncode != 0
        except subprocess.TimeoutExpired:
            failures += 1  # deadlock
    return failures > 0


def test_ring_model_detects_missing_consumer_free(tmp_path):
    assert _mutant_fails(tmp_path, "      w.store(0, std::memory_order_relaxed);  // free (same address: after the read)\n",
                         "", "ring_nofree"), "the model accepted a consumer that never frees a slot"


def test_ring_model_detects_producer_not_waiting(tmp_path):
    assert _mutant_fails(tmp_path, "        while (w.load(std::memory_order_relaxed) != 0) std::this_thread::yield();",
                         "        ;", "ring_nowait"), "the model accepted a producer that overwrites unconsumed records"
