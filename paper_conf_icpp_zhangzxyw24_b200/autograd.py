"""torch.autograd pairing of the two C-ABI calls: the paper's training
usage (§5.6; §6.3) runs the forward convolution and the
backward-data pass with Im2col-Winograd kernels: dX = deconv(dY, W), the same KRSC filter,
its 180-degree rotation folded into the filter transform. Both directions run in
libi2cw.so (conv2d_nhwc / deconv2d_nhwc); this module is argument plumbing only.

Backward-filter (dW = a correlation of X with dY, a filter as large as the output) is not a
small-filter convolution and is outside the method: requesting it raises.
"""
from __future__ import annotations

import torch

from . import conv2d_nhwc, conv3d_ndhwc, deconv2d_nhwc, deconv3d_ndhwc


class Conv2dNHWC(torch.autograd.Function):
    """y = conv(x, w, pad) in NHWC / KRSC; grad_x = deconv(grad_y, w, pad) (the exact adjoint:
    deconv(., w, pad) maps [N,P,Q,K] back to [N,H,W,C])."""

    @staticmethod
    def forward(ctx, x, w, pad_h: int, pad_w: int):
        ctx.save_for_backward(w)
        ctx.pad = (pad_h, pad_w)
        return conv2d_nhwc(x.contiguous(), w.contiguous(), pad_h, pad_w)

    @staticmethod
    def backward(ctx, grad_y):
        (w,) = ctx.saved_tensors
        if ctx.needs_input_grad[1]:
            raise NotImplementedError("i2cw: backward-filter (dW) is outside Im2col-Winograd; "
                                      "detach the filter or compute dW elsewhere")
        grad_x = None
        if ctx.needs_input_grad[0]:
            grad_x = deconv2d_nhwc(grad_y.contiguous(), w, ctx.pad[0], ctx.pad[1])
        return grad_x, None, None, None


def conv2d(x: torch.Tensor, w: torch.Tensor, pad_h: int, pad_w: int) -> torch.Tensor:
    """Differentiable (w.r.t. x) fused Im2col-Winograd convolution, NHWC x, KRSC w."""
    return Conv2dNHWC.apply(x, w, pad_h, pad_w)


class Conv3dNDHWC(torch.autograd.Function):
    """3D: y = conv3d(x, w, pad) in NDHWC / KTRSC; grad_x = deconv3d(grad_y, w, pad)."""

    @staticmethod
    def forward(ctx, x, w, pad_d: int, pad_h: int, pad_w: int):
        ctx.save_for_backward(w)
        ctx.pad = (pad_d, pad_h, pad_w)
        return conv3d_ndhwc(x.contiguous(), w.contiguous(), pad_d, pad_h, pad_w)

    @staticmethod
    def backward(ctx, grad_y):
        (w,) = ctx.saved_tensors
        if ctx.needs_input_grad[1]:
            raise NotImplementedError("i2cw: backward-filter (dW) is outside Im2col-Winograd; "
                                      "detach the filter or compute dW elsewhere")
        grad_x = None
        if ctx.needs_input_grad[0]:
            grad_x = deconv3d_ndhwc(grad_y.contiguous(), w, *ctx.pad)
        return grad_x, None, None, None, None


def conv3d(x: torch.Tensor, w: torch.Tensor, pad_d: int, pad_h: int, pad_w: int) -> torch.Tensor:
    """Differentiable (w.r.t. x) 3D fused Im2col-Winograd convolution, NDHWC x, KTRSC w."""
    return Conv3dNDHWC.apply(x, w, pad_d, pad_h, pad_w)
