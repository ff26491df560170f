"""Shared test helpers: device buffers, sentinel-filled outputs, one-call runs."""
import numpy as np
import torch

from paper_conf_isca_waddenlgss14_b200 import rmt

SENTINEL = 0xFFFFFFFF
VARIANTS = ("none",) + rmt.RMT_VARIANTS


def dev(a: np.ndarray) -> torch.Tensor:
    """numpy -> device tensor with the same bytes (u32 stored as int32)."""
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint32:
        a = a.view(np.int32)
    elif a.dtype == np.uint16:
        a = a.view(np.int16)
    elif a.dtype == np.uint64:
        a = a.view(np.int64)
    return torch.from_numpy(a.copy()).cuda()


def out_like(nbytes: int) -> torch.Tensor:
    """Sentinel-filled (all 0xFF bytes) device buffer, so an uncommitted store is visible."""
    t = torch.empty(nbytes // 4, dtype=torch.int32, device="cuda")
    t.fill_(-1)
    return t


def host(t: torch.Tensor, dtype) -> np.ndarray:
    return t.cpu().numpy().view(dtype)


def run(kernel, variant, tensors, n, dims=(), ws=None):
    """Launch once on the current stream; return the error count."""
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    if ws is None:
        ws = rmt.make_workspace(kernel, variant, n, dims)
    rmt.launch(kernel, variant, tensors, n, err, dims=dims, workspace=ws)
    torch.cuda.synchronize()
    return int(err.item())
