"""Helpers shared by the GPU tests (no method arithmetic)."""
import numpy as np

from workloads import bits_to_f64

TOL_MAX = 2e-2   # north_star: max-abs error vs the fp64 oracle
TOL_MEAN = 2e-3  # north_star: mean-abs error


def to_device(bits: np.ndarray, dtype: str = "bf16"):
    import torch
    t = torch.from_numpy(np.ascontiguousarray(bits).view(np.int16))
    t = t.view(torch.bfloat16 if dtype == "bf16" else torch.float16)
    return t.cuda()


def from_device(t) -> np.ndarray:
    """16-bit device tensor -> fp64 numpy (exact)."""
    import torch
    bits = t.detach().contiguous().view(torch.int16).cpu().numpy().view(np.uint16)
    return bits_to_f64(bits, "bf16" if t.dtype == torch.bfloat16 else "fp16")


def err_stats(got: np.ndarray, ref: np.ndarray):
    e = np.abs(got - ref)
    return float(e.max()), float(e.mean())
