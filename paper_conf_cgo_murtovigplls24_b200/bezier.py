"""Thin torch-facing wrappers over xs_bezier_surface / xs_bezier_blend (include/xs.h;
PAPER.md Listing 2).  Argument marshalling only: the loop, the powers
and the contraction all run in csrc/bezier.cu."""
from __future__ import annotations

import torch

from . import _xs

_DT = {torch.float64: _xs.XS_F64, torch.float32: _xs.XS_F32}


def _variant(v) -> int:
    return _xs.BZ_NAMES[v] if isinstance(v, str) else int(v)


def _stream_ptr(stream) -> int | None:
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def bezier_surface(ctrl: torch.Tensor, res_i: int, res_j: int, variant="T", out: torch.Tensor | None = None,
                   stream=None) -> torch.Tensor:
    """Evaluate the res_i x res_j surface of the control net ctrl[(ni+1), (nj+1), 3]
    (a CUDA tensor, float64 or float32); returns out[res_i, res_j, 3] of ctrl's dtype."""
    if not ctrl.is_cuda or ctrl.dim() != 3 or ctrl.shape[2] != 3 or ctrl.dtype not in _DT:
        raise ValueError("ctrl must be a CUDA float64/float32 tensor of shape [ni+1, nj+1, 3]")
    ctrl = ctrl.contiguous()
    if out is None:
        out = torch.empty((res_i, res_j, 3), dtype=ctrl.dtype, device=ctrl.device)
    if out.dtype != ctrl.dtype or not out.is_contiguous() or out.numel() != res_i * res_j * 3:
        raise ValueError("out must be a contiguous [res_i, res_j, 3] tensor of ctrl's dtype")
    with torch.cuda.device(ctrl.device):
        _xs.xs_bezier_surface(ctrl.shape[0] - 1, ctrl.shape[1] - 1, res_i, res_j, _DT[ctrl.dtype],
                              _variant(variant), ctrl, out, _stream_ptr(stream))
    return out


def bezier_blend(k: torch.Tensor, n: torch.Tensor, mu: torch.Tensor | None = None, variant="M",
                 dtype=torch.float64, stream=None) -> torch.Tensor:
    """out[t] = BezierBlend(k[t], mu[t], n[t]), or the bare Listing-2 loop when mu is None."""
    k = k.to(torch.int32).contiguous()
    n = n.to(torch.int32).contiguous()
    if mu is not None:
        mu = mu.to(dtype).contiguous()
    out = torch.empty(k.shape, dtype=dtype, device=k.device)
    with torch.cuda.device(k.device):
        _xs.xs_bezier_blend(k.numel(), k, n, mu, _DT[dtype], _variant(variant), out, _stream_ptr(stream))
    return out
