"""Shared helpers for the -m gpu tests: move seeded workloads to the device
and run the oracle on the same inputs."""
import numpy as np
import torch

from oracle import spmv as ospmv


def to_dev(A, device="cuda:0"):
    return (torch.from_numpy(np.ascontiguousarray(A.row_ptr, np.int32)).to(device),
            torch.from_numpy(np.ascontiguousarray(A.col, np.int32)).to(device),
            torch.from_numpy(np.ascontiguousarray(A.val, np.float32)).to(device))


def vec(x, device="cuda:0"):
    return torch.from_numpy(np.ascontiguousarray(x, np.float32)).to(device)


def oracle_spmv(A, x):
    return ospmv.spmv(A.row_ptr, A.col, A.val, x), ospmv.spmv_abs(A.row_ptr, A.col, A.val, x)


def spmv_err(A, x, y_dev):
    ys, d = oracle_spmv(A, x)
    return ospmv.rel_error(y_dev.cpu().numpy(), ys, d)


def unit_slices(n_rows):
    return [(u * 256, min(n_rows, (u + 1) * 256)) for u in range((n_rows + 255) // 256)]
