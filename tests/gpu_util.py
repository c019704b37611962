"""Helpers for -m gpu tests: column-major host arrays <-> flat device buffers (torch is
plumbing only: it owns device memory and streams; all compute is in libxk.so)."""
import numpy as np


def to_dev(a):
    import torch
    return torch.from_numpy(np.asfortranarray(a).ravel(order="F").copy()).to("cuda")


def from_dev(t, ld, ncols):
    return t.cpu().numpy().reshape((ld, ncols), order="F")


def stream_ptr():
    import torch
    return torch.cuda.current_stream().cuda_stream


def device_map(G):
    """Logical GPU -> physical device: distinct devices when the box has at least G of them
    (real NVLink peer copies), else all on device 0 (logical-device mode)."""
    import torch
    n = torch.cuda.device_count()
    return list(range(G)) if n >= G else [0] * G
