"""Operator tables of the paper's workloads (synthetic shapes only; no
weights).  ResNet-50 / ResNet-18 / MobileNet-V2 follow torchvision (readings
A16, A17); BERT-base GEMMs at seq 512 (A15).  Paper: E2E networks P:1590-1603,
single-operator sampling P:1546-1554."""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class ConvShape:
    name: str
    C: int
    H: int
    W: int
    K: int
    R: int
    S: int
    stride: int
    pad: int
    groups: int = 1

    def out_hw(self):
        return ((self.H + 2 * self.pad - self.R) // self.stride + 1,
                (self.W + 2 * self.pad - self.S) // self.stride + 1)

    def flops(self, N: int) -> float:
        Ho, Wo = self.out_hw()
        return 2.0 * N * self.K * Ho * Wo * (self.C // self.groups) * self.R * self.S

    def min_bytes(self, N: int, esize: int = 2) -> float:
        """algorithmic bytes: read x and w once, write y once"""
        Ho, Wo = self.out_hw()
        return esize * (N * self.C * self.H * self.W + self.K * (self.C // self.groups) * self.R * self.S
                        + N * self.K * Ho * Wo)


def _c(name, C, H, K, R, s, p=None, groups=1):
    return ConvShape(name, C, H, H, K, R, R, s, R // 2 if p is None else p, groups)


# 23 unique conv shapes of torchvision ResNet-50 v1.5
RESNET50 = [
    _c("conv1", 3, 224, 64, 7, 2, 3),
    _c("l1.1x1a", 64, 56, 64, 1, 1),
    _c("l1.3x3", 64, 56, 64, 3, 1),
    _c("l1.1x1b", 64, 56, 256, 1, 1),
    _c("l1.1x1c", 256, 56, 64, 1, 1),
    _c("l2.1x1a", 256, 56, 128, 1, 1),
    _c("l2.3x3s2", 128, 56, 128, 3, 2),
    _c("l2.1x1b", 128, 28, 512, 1, 1),
    _c("l2.ds", 256, 56, 512, 1, 2),
    _c("l2.1x1c", 512, 28, 128, 1, 1),
    _c("l2.3x3", 128, 28, 128, 3, 1),
    _c("l3.1x1a", 512, 28, 256, 1, 1),
    _c("l3.3x3s2", 256, 28, 256, 3, 2),
    _c("l3.1x1b", 256, 14, 1024, 1, 1),
    _c("l3.ds", 512, 28, 1024, 1, 2),
    _c("l3.1x1c", 1024, 14, 256, 1, 1),
    _c("l3.3x3", 256, 14, 256, 3, 1),
    _c("l4.1x1a", 1024, 14, 512, 1, 1),
    _c("l4.3x3s2", 512, 14, 512, 3, 2),
    _c("l4.1x1b", 512, 7, 2048, 1, 1),
    _c("l4.ds", 1024, 14, 2048, 1, 2),
    _c("l4.1x1c", 2048, 7, 512, 1, 1),
    _c("l4.3x3", 512, 7, 512, 3, 1),
]


def resnet18_chain(img: int = 224):
    """ResNet-18 conv chain (torchvision): conv1 7x7 s2 + maxpool 3x3 s2,
    4 stages x 2 BasicBlocks (3x3 convs, 1x1 s2 downsample on stages 2-4),
    folded BN + ReLU, residual adds.  Returns a list of ops:
      ("conv", ConvShape, input_id, residual_id or None, relu, out_id)
      ("maxpool", k, s, p, input_id, out_id)
    ids name activation tensors."""
    ops = [("conv", _c("conv1", 3, img, 64, 7, 2, 3), "img", None, True, "c1"),
           ("maxpool", 3, 2, 1, "c1", "p1")]
    h1 = (img + 6 - 7) // 2 + 1
    cur, C, H = "p1", 64, (h1 + 2 - 3) // 2 + 1
    for stage, (K, stride) in enumerate([(64, 1), (128, 2), (256, 2), (512, 2)]):
        for blk in range(2):
            s = stride if blk == 0 else 1
            pre = f"s{stage}b{blk}"
            Ho = (H + 2 - 3) // s + 1
            ops.append(("conv", _c(pre + ".a", C, H, K, 3, s, 1), cur, None, True, pre + ".a"))
            if s != 1 or C != K:
                ops.append(("conv", _c(pre + ".ds", C, H, K, 1, s, 0), cur, None, False, pre + ".ds"))
                short = pre + ".ds"
            else:
                short = cur
            ops.append(("conv", _c(pre + ".b", K, Ho, K, 3, 1, 1), pre + ".a", short, True, pre + ".out"))
            cur, C, H = pre + ".out", K, Ho
    return ops


def mobilenet_v2_chain(img: int = 224):
    """MobileNet-V2 (torchvision, width 1.0, 224): stem 3x3 s2 -> 17
    inverted-residual blocks (expand 1x1 + ReLU6, depthwise 3x3 + ReLU6,
    project 1x1 linear, residual add when stride 1 and C_in == C_out) ->
    1x1 1280 conv.  52 convs, 17 depthwise.  Same op encoding as
    resnet18_chain (relu flag means ReLU6 here)."""
    cfg = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1), (6, 160, 3, 2),
           (6, 320, 1, 1)]
    ops = [("conv", _c("stem", 3, img, 32, 3, 2, 1), "img", None, True, "stem")]
    cur, C, H = "stem", 32, (img + 2 - 3) // 2 + 1
    bi = 0
    for t, c, n, s in cfg:
        for i in range(n):
            stride = s if i == 0 else 1
            hid = C * t
            pre = f"b{bi}"
            src = cur
            if t != 1:
                ops.append(("conv", _c(pre + ".exp", C, H, hid, 1, 1, 0), src, None, True, pre + ".exp"))
                src = pre + ".exp"
            Ho = (H + 2 - 3) // stride + 1
            ops.append(("conv", _c(pre + ".dw", hid, H, hid, 3, stride, 1, groups=hid), src, None, True,
                        pre + ".dw"))
            res = cur if (stride == 1 and C == c) else None
            ops.append(("conv", _c(pre + ".proj", hid, Ho, c, 1, 1, 0), pre + ".dw", res, False, pre + ".out"))
            cur, C, H = pre + ".out", c, Ho
            bi += 1
    ops.append(("conv", _c("head", C, H, 1280, 1, 1, 0), cur, None, True, "head"))
    return ops


# BERT-base GEMMs at seq 512 (reading A15): (name, K, N)
BERT_GEMMS = [("qkv/out 768x768", 768, 768), ("ffn1 768x3072", 768, 3072), ("ffn2 3072x768", 3072, 768)]
