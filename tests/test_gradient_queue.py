"""Gradient queue plumbing (C2): flat buffer layout, Layer-Chunk Table
source, per-layer update hooks; on the GPU, chained == unchained training."""

import pytest
import torch
from torch import nn

from paper_conf_hpca_sanghoonsk23_b200 import workloads
from paper_conf_hpca_sanghoonsk23_b200.gradient_queue import attach_gradient_queue, layer_groups

torchvision = pytest.importorskip("torchvision")


@pytest.mark.parametrize("name", ["resnet50", "vgg16"])
def test_layer_groups_match_workload_tables(name):
    """The queue's layers are the workloads.py layers (54 for ResNet-50, 16 for VGG-16)."""
    m = getattr(torchvision.models, name)(weights=None)
    groups, leaders = layer_groups(m)
    assert [sum(p.numel() for p in g) for g in groups] == workloads.WORKLOADS[name]
    assert len(leaders) == len(groups)
    assert all(isinstance(x, (nn.Conv2d, nn.Linear)) for x in leaders)


def test_registration_order_is_forward_order_resnet50():
    """Gates are enqueued in call order, so leader pre-hooks must fire in layer order."""
    m = torchvision.models.resnet50(weights=None)
    _, leaders = layer_groups(m)
    seen = []
    hs = [x.register_forward_pre_hook(lambda mod, _i, l=l: seen.append(l))
          for l, x in enumerate(leaders)]
    with torch.no_grad():
        m.eval()(torch.zeros(1, 3, 64, 64))
    for h in hs:
        h.remove()
    assert seen == list(range(len(leaders)))


def _tiny():
    torch.manual_seed(3)
    return nn.Sequential(nn.Conv2d(3, 8, 3), nn.BatchNorm2d(8), nn.ReLU(), nn.Conv2d(8, 4, 3),
                         nn.BatchNorm2d(4), nn.Flatten(), nn.Linear(4 * 4 * 4, 5))


def test_flat_buffer_views_and_layer_ends():
    m = _tiny()
    gq = attach_gradient_queue(m)
    sizes = [8 * 3 * 9 + 8 + 16, 4 * 8 * 9 + 4 + 8, 64 * 5 + 5]
    assert gq.layer_ends == [sizes[0], sizes[0] + sizes[1], sum(sizes)]
    assert gq.flat.numel() == sum(p.numel() for p in m.parameters())
    off = 0
    for p in m.parameters():          # registration order = flat order
        assert p.grad.data_ptr() == gq.flat[off:].data_ptr()
        off += p.numel()
    # backward writes the queue in place
    x = torch.randn(2, 3, 8, 8)
    m(x).sum().backward()
    assert gq.flat.abs().sum() > 0
    for p in m.parameters():
        assert p.grad.data_ptr() >= gq.flat.data_ptr()
    gq.remove()


def test_update_hook_applies_averaged_sgd_per_layer():
    """The pre-hook of layer l applies p -= lr/P * g (R14: the library sums)."""
    m = _tiny()
    gq = attach_gradient_queue(m, lr=0.5, world_size=4)
    x = torch.randn(2, 3, 8, 8)
    m(x).sum().backward()
    before = [p.detach().clone() for p in m.parameters()]
    grads = [p.grad.clone() for p in m.parameters()]
    gq.update = True
    with torch.no_grad():
        m(x)
    for b, g, p in zip(before, grads, m.parameters()):
        assert torch.equal(p.detach(), b - 0.125 * g)
    gq.remove()


@pytest.mark.gpu
@pytest.mark.parametrize("kind", ["single", "double"])
def test_chained_training_equals_unchained(kind):
    """CC vs C1 (chaining changes timing, never values): three data-parallel
    iterations over P=4 loopback ranks give bitwise-identical parameters whether the
    next forward waits for the whole AllReduce or per layer on its gate."""
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    torch.backends.cudnn.deterministic = True
    torch.backends.cudnn.benchmark = False
    P, rr = 4, 1
    finals = {}
    for chained in (False, True):
        m = _tiny().cuda()
        gq = attach_gradient_queue(m, lr=0.1, world_size=P, local_rank=rr)
        gq.update = True
        others = [torch.zeros_like(gq.flat) for _ in range(P - 1)]
        bufs = others[:rr] + [gq.flat] + others[rr:]
        comp, comm = torch.cuda.Stream(), torch.cuda.Stream()
        ccube.init_loopback(P, kind, 256)
        try:
            ccube.set_channels(2)
            gq.set_layers()
            gq.chained = chained
            g = torch.Generator().manual_seed(9)
            for it in range(3):
                x = torch.randn(16, 3, 8, 8, generator=g).cuda()
                with torch.cuda.stream(comp):
                    loss = m(x).square().mean()
                    comp.wait_stream(comm)
                    gq.zero_()
                    loss.backward()
                    for r, o in enumerate(others):
                        o.copy_(gq.flat * (r + 2))   # distinct emulated replica gradients
                comm.wait_stream(comp)
                ccube.allreduce_tree_local(bufs, stream=comm)
                if not chained:
                    comp.wait_stream(comm)
            with torch.cuda.stream(comp), torch.no_grad():
                m(torch.zeros(1, 3, 8, 8, device="cuda"))   # consumes the last AllReduce
            torch.cuda.synchronize()
        finally:
            gq.remove()
            ccube.finalize()
        finals[chained] = [p.detach().cpu() for p in m.parameters()]
    for a, b in zip(finals[False], finals[True]):
        assert torch.equal(a, b)


def test_views_keep_channels_last_strides():
    m = torchvision.models.resnet50(weights=None).to(memory_format=torch.channels_last)
    strides = {n: p.stride() for n, p in m.named_parameters()}
    gq = attach_gradient_queue(m)
    for n, p in m.named_parameters():   # strides of size-1 dims carry no layout
        assert p.grad.shape == p.shape
        assert [s for s, k in zip(p.grad.stride(), p.shape) if k > 1] == \
            [s for s, k in zip(strides[n], p.shape) if k > 1]
    gq.remove()


def test_fused_mode_moves_weights_into_flat_buffer():
    m = _tiny()
    before = [p.detach().clone() for p in m.parameters()]
    gq = attach_gradient_queue(m, lr=0.1, world_size=2, fused_sgd=True)
    off = 0
    for b, p in zip(before, m.parameters()):
        assert torch.equal(p.detach(), b)
        assert p.data_ptr() == gq.flat_w[off:].data_ptr()
        off += p.numel()
    # the pre-hook no longer updates (the AllReduce kernel does)
    x = torch.randn(2, 3, 8, 8)
    m(x).sum().backward()
    gq.update = True
    with torch.no_grad():
        m(x)
    for b, p in zip(before, m.parameters()):
        assert torch.equal(p.detach(), b)
    gq.remove()


@pytest.mark.gpu
def test_fused_chained_training_equals_fused_unchained():
    """f2 + C2: with the update fused into the AllReduce, chaining still changes
    timing only."""
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    torch.backends.cudnn.deterministic = True
    torch.backends.cudnn.benchmark = False
    P, rr = 4, 2
    finals = {}
    for chained in (False, True):
        m = _tiny().cuda()
        gq = attach_gradient_queue(m, lr=0.1, world_size=P, local_rank=rr, fused_sgd=True)
        others = [torch.zeros_like(gq.flat) for _ in range(P - 1)]
        bufs = others[:rr] + [gq.flat] + others[rr:]
        ow = [gq.flat_w.clone() for _ in range(P - 1)]
        wts = ow[:rr] + [gq.flat_w] + ow[rr:]
        comp, comm = torch.cuda.Stream(), torch.cuda.Stream()
        ccube.init_loopback(P, "double", 256)
        try:
            ccube.set_channels(2)
            gq.set_layers(weights=wts)
            gq.chained = chained
            g = torch.Generator().manual_seed(4)
            for it in range(3):
                x = torch.randn(16, 3, 8, 8, generator=g).cuda()
                with torch.cuda.stream(comp):
                    loss = m(x).square().mean()
                    comp.wait_stream(comm)
                    gq.zero_()
                    loss.backward()
                    for r, o in enumerate(others):
                        o.copy_(gq.flat * (r + 2))
                comm.wait_stream(comp)
                ccube.allreduce_tree_local(bufs, stream=comm)
                if not chained:
                    comp.wait_stream(comm)
            with torch.cuda.stream(comp), torch.no_grad():
                m(torch.zeros(1, 3, 8, 8, device="cuda"))
            torch.cuda.synchronize()
        finally:
            gq.remove()
            ccube.finalize()
        finals[chained] = [p.detach().cpu() for p in m.parameters()]
        assert not torch.equal(finals[chained][0], _tiny().state_dict()["0.weight"])
    for a, b in zip(finals[False], finals[True]):
        assert torch.equal(a, b)
