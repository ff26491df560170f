"""Reference rates on this GPU for context: copy bandwidth (torch clone), CUB
inclusive scan (torch.cumsum) and reduction (torch.sum) at the suite's sizes.
usage: ref_rates.py [LOG2N]"""
import sys, statistics
import torch

n = 1 << (int(sys.argv[1]) if len(sys.argv) > 1 else 26)
x = torch.randint(0, 256, (n,), dtype=torch.int32, device="cuda")


def t(f, reps=20):
    for _ in range(3):
        f()
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); f(); e.record(); torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    return statistics.median(ts)


y = torch.empty_like(x)
for name, f, bytes_ in [("copy", lambda: y.copy_(x), 8 * n),
                        ("cumsum_i32(CUB)", lambda: torch.cumsum(x, 0, out=y), 8 * n),
                        ("sum_i64", lambda: x.sum(dtype=torch.int64), 4 * n)]:
    ms = t(f)
    print(f"{name:18s} n=2^{n.bit_length()-1} {ms*1e3:8.1f} us  {bytes_/ms/1e6:8.1f} GB/s")
