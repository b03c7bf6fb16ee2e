"""The shared seeded generator: determinism, chunking independence, distribution."""

import numpy as np
import pytest

from paper_conf_hpca_sanghoonsk23_b200 import inputs, workloads


@pytest.mark.parametrize("dtype", ["float32", "bfloat16", "int32"])
def test_value_depends_only_on_seed_rank_element(dtype):
    a = inputs.gradients(3, 10000, dtype)
    b = inputs.gradients(3, 10000, dtype, lo=4000, hi=7000)
    assert np.array_equal(a[4000:7000], b)
    assert np.array_equal(a, inputs.gradients(3, 10000, dtype))
    assert not np.array_equal(a, inputs.gradients(4, 10000, dtype))


def test_normal_with_layer_scales():
    ends = [50000, 100000]
    x = inputs.gradients_f32(0, 100000, layer_ends=ends).astype(np.float64)
    assert abs(x[:50000].std() - 1.0) < 0.02 and abs(x[50000:].std() - 0.5) < 0.01
    assert abs(x[:50000].mean()) < 0.02


def test_int32_ranges():
    x = inputs.gradients_i32(0, 200000)
    assert x.min() >= -(1 << 24) and x.max() < (1 << 24)
    y = inputs.gradients_i32(0, 200000, full_range=True)
    assert y.min() < -(1 << 30) and y.max() > (1 << 30)


def test_workload_totals():
    assert workloads.total_elems("resnet50") == 25557032
    assert len(workloads.RESNET50_LAYER_ELEMS) == 54
    assert workloads.total_elems("vgg16") == 138357544
    assert len(workloads.VGG16_LAYER_ELEMS) == 16


def test_workloads_match_torchvision():
    tv = pytest.importorskip("torchvision")
    import torch
    for name, ctor in (("resnet50", tv.models.resnet50), ("vgg16", tv.models.vgg16)):
        m = ctor(weights=None)
        mods = dict(m.named_modules())
        groups = []
        for n, p in m.named_parameters():
            mod, leaf = n.rsplit(".", 1)
            if isinstance(mods[mod], (torch.nn.Conv2d, torch.nn.Linear)) and leaf == "weight":
                groups.append(p.numel())
            else:
                groups[-1] += p.numel()
        assert groups == workloads.WORKLOADS[name]


def test_zfnet_layers_match_workload_table():
    """The ZFNet-like net (f4) has the published layer sizes: 8 layers,
    62,357,608 parameters, and its queue layers are ZFNET_LAYER_ELEMS."""
    from paper_conf_hpca_sanghoonsk23_b200.gradient_queue import layer_groups
    m = workloads.zfnet()
    groups, _ = layer_groups(m)
    assert [sum(p.numel() for p in g) for g in groups] == workloads.WORKLOADS["zfnet"]
    assert workloads.total_elems("zfnet") == 62_357_608
