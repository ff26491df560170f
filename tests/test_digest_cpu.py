"""Host-side check of the Inter-Group record digest (-m "not gpu"; reading
R-C-Q2): tests/model/digest_check.cu includes rmt_device.cuh and verifies that
rec_digest changes for every single-bit flip of the key or of any stored word,
and for any change confined to one word, over random records of 1, 2 and 4
words; and that a non-storing lane's digest is the compile-time constant."""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)


def test_digest_detects_every_single_word_change(tmp_path):
    exe = str(tmp_path / "digest_check")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-I", os.path.join(ROOT, "include"), "-I",
                           os.path.join(ROOT, "paper_conf_isca_waddenlgss14_b200", "csrc"),
                           os.path.join(HERE, "model", "digest_check.cu"), "-o", exe])
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0 and r.stdout.startswith("ok"), r.stdout + r.stderr
