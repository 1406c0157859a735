"""Shared test helpers (marshalling only — no layout arithmetic)."""
import numpy as np

_SIGNED = {1: np.uint8, 2: np.int16, 4: np.int32, 8: np.int64}
_UNSIGNED = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}


def to_device(a: np.ndarray):
    """Copy a numpy bit-pattern array to a CUDA tensor (signed view; same bits)."""
    import torch
    a = np.ascontiguousarray(a)
    return torch.from_numpy(a.view(_SIGNED[a.itemsize])).cuda()


def from_device(t, elem_bytes: int) -> np.ndarray:
    return t.cpu().numpy().view(_UNSIGNED[elem_bytes])


def empty_device(n: int, elem_bytes: int):
    import torch
    dt = {1: torch.uint8, 2: torch.int16, 4: torch.int32, 8: torch.int64}[elem_bytes]
    return torch.empty(n, dtype=dt, device="cuda")


def gpu_available() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
