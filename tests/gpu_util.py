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
