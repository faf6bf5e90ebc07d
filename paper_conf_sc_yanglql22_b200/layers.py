"""GNN layer op on the prepared mini-batch: g-SpMM mean aggregation
over the sub-graph CSR, forward and backward in libwg.so, wrapped as a torch.autograd
Function ("we make use of the automatic differentiation module in PyTorch", L94)."""

import ctypes

import torch

from ._lib import check, lib


def _p(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def _s():
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


def spmm_mean_forward(row_ptr, sub_col, x, n_rows=None, n_rows_dev=None):
    """Y[t] = mean of x[sub_col[e]] over row t's edges.  x: float32 [*, D], D % 4 == 0."""
    n = row_ptr.numel() - 1 if n_rows is None else n_rows
    # with a device row count the kernel writes only rows below it: the rest read as 0
    alloc = torch.empty if n_rows_dev is None else torch.zeros
    y = alloc((n, x.shape[1]), dtype=torch.float32, device=x.device)
    check(lib().wg_spmm_mean_forward(_p(row_ptr), n, _p(n_rows_dev), _p(sub_col), _p(x.contiguous()), x.shape[0],
                                     x.shape[1], _p(y), _s()))
    return y


def spmm_mean_backward(row_ptr, sub_col, dup, dy, n_x_rows, n_rows=None, n_rows_dev=None):
    n = row_ptr.numel() - 1 if n_rows is None else n_rows
    dx = torch.empty((n_x_rows, dy.shape[1]), dtype=torch.float32, device=dy.device)
    check(lib().wg_spmm_mean_backward(_p(row_ptr), n, _p(n_rows_dev), _p(sub_col), _p(dup), _p(dy.contiguous()),
                                      dy.shape[1], _p(dx), n_x_rows, _s()))
    return dx


class SpMMMean(torch.autograd.Function):
    """autograd wrapper: forward = g-SpMM mean on the CSR, backward = atomics on the same
    CSR with the duplicate-count store fast path.  ``row_ptr`` may be a pipeline's untrimmed
    [capacity + 1] buffer when ``n_rows_dev`` (the device row count, e.g. the previous hop's
    num_unique) is given: rows past it are left untouched (zero in the output)."""

    @staticmethod
    def forward(ctx, x, row_ptr, sub_col, dup, n_rows_dev=None):
        ctx.save_for_backward(row_ptr, sub_col, dup, n_rows_dev)
        ctx.n_x = x.shape[0]
        return spmm_mean_forward(row_ptr, sub_col, x, n_rows_dev=n_rows_dev)

    @staticmethod
    def backward(ctx, dy):
        row_ptr, sub_col, dup, n_rows_dev = ctx.saved_tensors
        return spmm_mean_backward(row_ptr, sub_col, dup, dy, ctx.n_x, n_rows_dev=n_rows_dev), None, None, None, None
