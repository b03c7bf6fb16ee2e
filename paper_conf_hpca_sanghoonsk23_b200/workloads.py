"""Gradient-set shapes of the paper's workloads (ZFNet, VGG-16, ResNet-50).

Only SHAPES are used (no weights, no datasets).  A "layer" is one conv or linear
module plus its batch-norm parameters, in forward (registration) order, i.e. the
granularity of the Layer-Chunk Table.  The lists were taken once from
``torchvision.models.resnet50(weights=None)`` / ``vgg16(weights=None)``
parameter shapes; ``tests/test_workloads.py`` re-derives them from torchvision
when it is importable.
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

WORKLOADS: Dict[str, List[int]] = {
    "resnet50": RESNET50_LAYER_ELEMS,
    "vgg16": VGG16_LAYER_ELEMS,
}


def layer_ends(name: str) -> List[int]:
    """Cumulative element offsets where each layer ends (forward order)."""
    return list(accumulate(WORKLOADS[name]))


def total_elems(name: str) -> int:
    return sum(WORKLOADS[name])
