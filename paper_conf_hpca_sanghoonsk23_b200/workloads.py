"""Gradient-set shapes of the paper's workloads (ZFNet, VGG-16, ResNet-50).

Only SHAPES are used (no weights, no datasets).  A "layer" is one conv or linear
module plus its batch-norm parameters, in forward (registration) order, i.e. the
granularity of the Layer-Chunk Table.  The ResNet-50 / VGG-16 lists were
taken once from ``torchvision.models.resnet50(weights=None)`` / ``vgg16(weights=None)``
parameter shapes; ``tests/test_inputs.py`` and ``tests/test_gradient_queue.py``
re-derive them from torchvision when it is importable.  ZFNet has no torchvision
model: ``zfnet()`` below builds a ZFNet-like net (Zeiler & Fergus's layer sizes)
whose parameter shapes give ``ZFNET_LAYER_ELEMS``.
"""

from itertools import accumulate
from typing import Dict, List

# 53 conv(+BN) layers + fc; 161 tensors; 25,557,032 parameters (fp32: 102,228,128 B)
RESNET50_LAYER_ELEMS: List[int] = [
    9536, 4224, 36992, 16896, 16896, 16512, 36992, 16896, 16512, 36992, 16896, 33024,
    147712, 66560, 132096, 65792, 147712, 66560, 65792, 147712, 66560, 65792, 147712,
    66560, 131584, 590336, 264192, 526336, 262656, 590336, 264192, 262656, 590336,
    264192, 262656, 590336, 264192, 262656, 590336, 264192, 262656, 590336, 264192,
    525312, 2360320, 1052672, 2101248, 1049600, 2360320, 1052672, 1049600, 2360320,
    1052672, 2049000,
]

# 13 conv + 3 linear layers; 32 tensors; 138,357,544 parameters (bf16: 276,715,088 B)
VGG16_LAYER_ELEMS: List[int] = [
    1792, 36928, 73856, 147584, 295168, 590080, 590080, 1180160, 2359808, 2359808,
    2359808, 2359808, 2359808, 102764544, 16781312, 4097000,
]

# 5 conv + 3 linear layers; 16 tensors; 62,357,608 parameters (fp32: 249,430,432 B)
ZFNET_LAYER_ELEMS: List[int] = [
    14208, 614656, 885120, 1327488, 884992, 37752832, 16781312, 4097000,
]

WORKLOADS: Dict[str, List[int]] = {
    "resnet50": RESNET50_LAYER_ELEMS,
    "vgg16": VGG16_LAYER_ELEMS,
    "zfnet": ZFNET_LAYER_ELEMS,
}


def zfnet(num_classes: int = 1000):
    """A ZFNet-like CNN (the paper's third network): AlexNet's layout with
    ZFNet's 7x7 stride-2 first conv and 5x5 stride-2 second conv, 224x224 inputs.
    Random init; only its shapes and compute profile are used (a synthetic
    workload for the chained iteration, f4)."""
    from torch import nn
    return nn.Sequential(
        nn.Conv2d(3, 96, 7, stride=2, padding=1), nn.ReLU(inplace=True),
        nn.MaxPool2d(3, stride=2, padding=1),
        nn.Conv2d(96, 256, 5, stride=2), nn.ReLU(inplace=True),
        nn.MaxPool2d(3, stride=2, padding=1),
        nn.Conv2d(256, 384, 3, padding=1), nn.ReLU(inplace=True),
        nn.Conv2d(384, 384, 3, padding=1), nn.ReLU(inplace=True),
        nn.Conv2d(384, 256, 3, padding=1), nn.ReLU(inplace=True),
        nn.MaxPool2d(3, stride=2),
        nn.AdaptiveAvgPool2d((6, 6)), nn.Flatten(),
        nn.Dropout(), nn.Linear(256 * 6 * 6, 4096), nn.ReLU(inplace=True),
        nn.Dropout(), nn.Linear(4096, 4096), nn.ReLU(inplace=True),
        nn.Linear(4096, num_classes),
    )


def layer_ends(name: str) -> List[int]:
    """Cumulative element offsets where each layer ends (forward order)."""
    return list(accumulate(WORKLOADS[name]))


def total_elems(name: str) -> int:
    return sum(WORKLOADS[name])
