"""Gradient queue (C2, §III-C): the model's gradients live in ONE flat buffer, laid
out in forward order, that the tree AllReduce reduces in place.  Because the tree
lands chunks in order (Obs #3), the buffer is a FIFO of reduced
gradient chunks and the next iteration's layer l may update and run its
forward as soon as the chunks holding its gradients have landed: a per-layer gate
``ccube_gradq_wait(l)`` (Enqueue Semaphore >= Layer-Chunk Table, P:L199-204,
P:L266) enqueued on the compute stream — no host synchronisation.

This module is the Python-side plumbing of that idea (argument marshalling and
PyTorch module hooks); the gate itself is the C-ABI call.  Layout:

* a *layer* is one conv/linear module plus the norm modules that follow it in
  registration order (``workloads.py``'s granularity); for torchvision's ResNet-50
  and VGG-16 registration order is forward order;
* ``flat`` holds every parameter's gradient, layer after layer; ``p.grad`` is a view
  into it, so autograd's backward writes the gradient queue directly;
* ``layer_ends[l]`` = element offset where layer l's gradients end (the source of the
  Layer-Chunk Table, ``ccube_gradq_set_layers``);
* a forward pre-hook on each layer's first module performs, on the current stream,
  (i) the gate (chained mode only) and (ii) the SGD update of that layer's
  parameters from the reduced (summed) gradients, ÷P for the average (R14);
* ``fused_sgd=True`` (NEXT f2): the parameters also live in one flat fp32 buffer
  (``flat_w``, same layout), ``p.data`` are views into it, and the AllReduce kernel
  itself applies w <- w - lr/P * g as each chunk lands (``ccube_gradq_set_sgd``);
  the gate then opens once the layer's WEIGHTS are updated and the pre-hook only
  enqueues the gate.
Views keep each parameter's own strides (e.g. channels_last conv weights), so
autograd and cuDNN see the layouts they would see without the queue.
"""

from typing import List, Optional, Tuple

import torch
from torch import nn

from . import ccube

_LEADERS = (nn.Conv1d, nn.Conv2d, nn.Conv3d, nn.Linear)


def layer_groups(model: nn.Module) -> Tuple[List[List[nn.Parameter]], List[nn.Module]]:
    """(parameter groups, leader modules): each conv/linear starts a new layer;
    modules without a leader of their own (norms) join the current one.  Forward
    order = registration order (checked for ResNet-50/VGG-16 by the tests)."""
    groups: List[List[nn.Parameter]] = []
    leaders: List[nn.Module] = []
    for m in model.modules():
        ps = [p for p in m.parameters(recurse=False) if p.requires_grad]
        if not ps:
            continue
        if isinstance(m, _LEADERS) or not groups:
            groups.append([])
            leaders.append(m)
        groups[-1].extend(ps)
    return groups, leaders


class GradientQueue:
    """Flat gradient buffer + per-layer gates for one model replica.

    ``local_rank`` selects the loopback rank whose Enqueue Semaphore gates this
    replica (one-process-per-GPU mode: leave it None)."""

    def __init__(self, model: nn.Module, lr: float = 0.0, world_size: int = 1,
                 local_rank: Optional[int] = None, dtype: torch.dtype = torch.float32,
                 fused_sgd: bool = False):
        self.model = model
        self.lr = lr
        self.world_size = world_size
        self.local_rank = local_rank
        self.groups, self.leaders = layer_groups(model)
        dev = next(model.parameters()).device
        sizes = [sum(p.numel() for p in g) for g in self.groups]
        self.numel = sum(sizes)
        self.flat = torch.zeros(self.numel, dtype=dtype, device=dev)
        self.fused_sgd = fused_sgd
        self.flat_w = None
        if fused_sgd:
            if dtype != torch.float32 or any(p.dtype != torch.float32 for g in self.groups
                                             for p in g):
                raise ValueError("the fused SGD update needs fp32 parameters and gradients")
            self.flat_w = torch.empty(self.numel, dtype=torch.float32, device=dev)
        self.layer_ends: List[int] = []
        off = 0
        for g in self.groups:
            for p in g:
                n = p.numel()
                p.grad = _dense_view(self.flat[off:off + n], p)
                if fused_sgd:
                    w = _dense_view(self.flat_w[off:off + n], p)
                    with torch.no_grad():
                        w.copy_(p.data)
                    p.data = w
                off += n
            self.layer_ends.append(off)
        self._grads = [[p.grad for p in g] for g in self.groups]
        self.chained = False   # gate each layer on the Enqueue Semaphore
        self.update = False    # apply the SGD step in the pre-hooks
        self._handles = [m.register_forward_pre_hook(self._hook(l))
                         for l, m in enumerate(self.leaders)]

    def set_layers(self, weights=None) -> None:
        """Hands the Layer-Chunk Table source to the library (after ccube_init); in
        fused mode also the weight buffers (``weights`` = one per rank hosted by this
        process, default ``[flat_w]``) and alpha = lr / P."""
        ccube.gradq_set_layers(self.layer_ends)
        if self.fused_sgd:
            ccube.gradq_set_sgd(weights if weights is not None else [self.flat_w],
                                self.lr / self.world_size)

    def _hook(self, l: int):
        def pre(_module, _inputs):
            if self.chained:
                s = torch.cuda.current_stream()
                if self.local_rank is None:
                    ccube.gradq_wait(l, stream=s)
                else:
                    ccube.gradq_wait_local(self.local_rank, l, stream=s)
            if self.update and self.lr != 0.0 and not self.fused_sgd:
                with torch.no_grad():
                    torch._foreach_add_([p for p in self.groups[l]], self._grads[l],
                                        alpha=-self.lr / self.world_size)
        return pre

    def zero_(self) -> None:
        """Backward accumulates into ``p.grad``: clear the queue once every layer's
        update has consumed it.  The caller orders this (and the backward) after the
        AllReduce itself, not just after the last gate: an interior rank's
        broadcast-down task still READS its buffer after the chunks landed there."""
        self.flat.zero_()

    def remove(self) -> None:
        for h in self._handles:
            h.remove()
        self._handles = []


def _dense_view(flat: torch.Tensor, p: torch.Tensor) -> torch.Tensor:
    """A view of ``flat`` (p.numel() elements) with p's shape and strides; p's
    layout must be dense (contiguous or a permutation of it, e.g. channels_last)."""
    if p.is_contiguous():
        return flat.view_as(p)
    order = sorted(range(p.dim()), key=lambda d: -p.stride(d))
    expect, dense = 1, True
    for d in reversed(order):
        if p.size(d) > 1 and p.stride(d) != expect:
            dense = False
        expect *= p.size(d)
    if not dense:
        raise ValueError("parameter layout is not dense")
    return flat.as_strided(p.shape, p.stride())


def attach_gradient_queue(model: nn.Module, **kw) -> GradientQueue:
    """Builds the flat gradient buffer, the ``p.grad`` views and the pre-hooks."""
    return GradientQueue(model, **kw)
