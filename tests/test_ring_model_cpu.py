"""CPU model of the inter-group queue protocol (-m "not gpu"; SURVEY 8(c)
"C-Q inter-group ring": a std::atomic model of the same protocol under stress).

tests/model/ring_model.cpp restates the protocol of rmt_device.cuh (V_INTER)
with C++ acquire/release atomics, one thread per CTA role and a pool of worker
threads standing in for the resident CTA slots.  Every configuration must finish
(no deadlock) with every record consumed once, in order, with its producer's
(pair, sequence) tag, and leave the control block zeroed -- at ring depth 1, 2,
4 and 8, one region (every pair hands the ring to the next) or several, and
down to 2 workers (the minimum residency the deadlock-freedom argument needs).
A mutant without the consumer's "free before waiting when S records are held"
rule must fail, and so must a mutant that publishes a group's flags in record
order behind one fence (a consumer that acquired the first flag may free a
later slot before that slot's flag store lands, leaving a stale "full" flag),
so the model can tell the difference.
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


def test_ring_model_detects_missing_consumer_free(tmp_path):
    text = open(SRC).read()
    rule = "      if (pend >= (unsigned)q.S) flush();\n"
    assert rule in text
    exe = _build(tmp_path, text.replace(rule, ""), "ring_mutant")
    try:
        r = subprocess.run([exe, "1", "2", "2", "16", "40", "1", "3"], capture_output=True, text=True, timeout=10)
        failed = r.returncode != 0
    except subprocess.TimeoutExpired:
        failed = True  # deadlock
    assert failed, "the model accepted a protocol without the consumer-side free rule"


def test_ring_model_detects_group_flags_published_in_order(tmp_path):
    text = open(SRC).read()
    fixed = """      for (unsigned l = 1; l < pend; ++l) {
        q.flag[slot(first + l)].store(pend - l, std::memory_order_relaxed);
        jitter(rng);
      }
      std::atomic_thread_fence(std::memory_order_seq_cst);  // fence.sc.gpu
      q.flag[slot(first)].store(pend, std::memory_order_relaxed);"""
    in_order = """      std::atomic_thread_fence(std::memory_order_seq_cst);  // fence.sc.gpu
      for (unsigned l = 0; l < pend; ++l) {
        q.flag[slot(first + l)].store(pend - l, std::memory_order_relaxed);
        jitter(rng);
      }"""
    assert fixed in text
    exe = _build(tmp_path, text.replace(fixed, in_order), "ring_in_order")
    failures = 0
    for seed in range(1, 4):
        try:
            r = subprocess.run([exe, "2", "1", "2", "48", "60", str(seed), "3"], capture_output=True, text=True, timeout=10)
            failures += r.returncode != 0
        except subprocess.TimeoutExpired:
            failures += 1  # a stale full flag: the producer waits forever
    assert failures > 0, "the model accepted group flags published first-record-first"
