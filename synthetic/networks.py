"""Conv layer tables of the paper's networks (workload definitions only).

* AlexNet: single-column (torchvision) shapes, reading G24 (P:L23 ref [11]),
  224x224 input (reading G26).
* ResNet-18 / ResNet-50: torchvision v1.5 shapes (stride on the 3x3 conv,
  reading G25), 224x224 input.

Each entry is one conv layer; `count` is not used -- repeated layers appear
repeatedly, in network order (forward order).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List


@dataclass(frozen=True)
class ConvLayer:
    name: str
    c: int
    h: int
    w: int
    k: int
    r: int
    s: int
    pad: int
    stride: int

    @property
    def p(self):
        return (self.h + 2 * self.pad - self.r) // self.stride + 1

    @property
    def q(self):
        return (self.w + 2 * self.pad - self.s) // self.stride + 1

    def flops(self, n):
        """Direct-convolution FLOPs of one direction at mini-batch n: 2 N K C R S P Q."""
        return 2 * n * self.k * self.c * self.r * self.s * self.p * self.q

    def key(self):
        return (self.c, self.h, self.w, self.k, self.r, self.s, self.pad, self.stride)


def alexnet() -> List[ConvLayer]:
    return [
        ConvLayer("conv1", 3, 224, 224, 64, 11, 11, 2, 4),
        ConvLayer("conv2", 64, 27, 27, 192, 5, 5, 2, 1),
        ConvLayer("conv3", 192, 13, 13, 384, 3, 3, 1, 1),
        ConvLayer("conv4", 384, 13, 13, 256, 3, 3, 1, 1),
        ConvLayer("conv5", 256, 13, 13, 256, 3, 3, 1, 1),
    ]


def resnet18() -> List[ConvLayer]:
    L = [ConvLayer("conv1", 3, 224, 224, 64, 7, 7, 3, 2)]
    h = 56
    cin = 64
    for stage, (cout, nblocks) in enumerate([(64, 2), (128, 2), (256, 2), (512, 2)], start=1):
        for b in range(nblocks):
            stride = 2 if (b == 0 and stage > 1) else 1
            hin = h
            hout = h // stride
            L.append(ConvLayer(f"layer{stage}.{b}.conv1", cin, hin, hin, cout, 3, 3, 1, stride))
            L.append(ConvLayer(f"layer{stage}.{b}.conv2", cout, hout, hout, cout, 3, 3, 1, 1))
            if stride != 1 or cin != cout:
                L.append(ConvLayer(f"layer{stage}.{b}.downsample", cin, hin, hin, cout, 1, 1, 0, stride))
            cin = cout
            h = hout
    return L


def resnet50() -> List[ConvLayer]:
    L = [ConvLayer("conv1", 3, 224, 224, 64, 7, 7, 3, 2)]
    h = 56
    cin = 64
    for stage, (width, nblocks) in enumerate([(64, 3), (128, 4), (256, 6), (512, 3)], start=1):
        cout = width * 4
        for b in range(nblocks):
            stride = 2 if (b == 0 and stage > 1) else 1
            hin = h
            hout = h // stride
            L.append(ConvLayer(f"layer{stage}.{b}.conv1", cin, hin, hin, width, 1, 1, 0, 1))
            L.append(ConvLayer(f"layer{stage}.{b}.conv2", width, hin, hin, width, 3, 3, 1, stride))
            L.append(ConvLayer(f"layer{stage}.{b}.conv3", width, hout, hout, cout, 1, 1, 0, 1))
            if b == 0:
                L.append(ConvLayer(f"layer{stage}.{b}.downsample", cin, hin, hin, cout, 1, 1, 0, stride))
            cin = cout
            h = hout
    return L


def network(name: str) -> List[ConvLayer]:
    return {"alexnet": alexnet, "resnet18": resnet18, "resnet50": resnet50}[name]()
