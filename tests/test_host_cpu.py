"""Host-side logic on CPU: the tune cache (conv and GEMM entries round trip,
the shipped cache covers the bench configurations), the chain tune keys, the
bench's CPU baseline sampling and its algorithmic-bytes bookkeeping."""
import json
import os

import pytest

import bench
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets, relayout_set, tunecache


def test_tune_cache_round_trip(tmp_path, monkeypatch):
    monkeypatch.setattr(tunecache, "_PATH", str(tmp_path / "tc.jsonl"))
    monkeypatch.setattr(tunecache, "_cache", None)
    L = nets.RESNET50[2]
    res = {"x": [("split", 1, [1, 64]), ("reorder", [0, 1, 3, 4, 2])], "w": [], "y": [("pad", 2, 1, 1)],
           "cfg": {"path": 1, "block_n": 64}, "best_us": 12.5}
    tunecache.store("conv2d", L, 32, res)
    tunecache.store_gemm(8192, 768, 768, {"path": 1, "block_n": 256, "b_nt": 256}, 17.9)
    monkeypatch.setattr(tunecache, "_cache", None)   # reload from disk
    hit = tunecache.lookup("conv2d", L, 32)
    assert hit["x"] == [("split", 1, [1, 64]), ("reorder", [0, 1, 3, 4, 2])] and hit["y"] == [("pad", 2, 1, 1)]
    assert hit["cfg"]["block_n"] == 64 and hit["us"] == 12.5
    assert tunecache.lookup("conv2d", L, 1) is None
    assert tunecache.lookup_gemm(8192, 768, 768)["b_nt"] == 256
    assert tunecache.lookup_gemm(8192, 768, 3072) is None


def test_shipped_caches_cover_the_bench_configurations():
    """every R50 layer at batch 32 and 1 has a tuned entry; the BERT GEMMs and
    the chain batches the bench runs have tuned kernel configurations"""
    for N in (32, 1):
        for L in nets.RESNET50:
            assert tunecache.lookup("conv2d", L, N) is not None, (L.name, N)
    for _, K, N in nets.BERT_GEMMS:
        assert tunecache.lookup_gemm(8192, N, K) is not None
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    with open(os.path.join(root, "chain_tune.json")) as f:
        keys = set(json.load(f))
    assert {"r18|N256", "r18|N128", "r18|N64", "r18|N32", "mv2|N16"} <= keys


def test_algorithmic_bytes_and_flops():
    """SURVEY 8d bookkeeping: conv FLOPs 2 N K Ho Wo C R S; minimum bytes
    elem (x + w + y); relayout bytes = elem (logical read + dst physical)"""
    L = nets.ConvShape("t", 64, 56, 56, 64, 3, 3, 1, 1, 1)
    assert L.out_hw() == (56, 56)
    assert L.flops(2) == 2 * 2 * 64 * 56 * 56 * 64 * 9
    assert L.min_bytes(2) == 2 * (2 * 64 * 56 * 56 + 64 * 64 * 9 + 2 * 64 * 56 * 56)

    class FakeLayout:
        def __init__(self, logical, phys):
            self.logical_shape, self.phys_numel = logical, phys
    assert relayout_set.alg_bytes(FakeLayout((2, 3), 6), FakeLayout((2, 3), 10), 2) == 2 * (6 + 10)


def test_cpu_baseline_sample_is_bounded():
    """bench's cpu_baseline runs the oracle on whole images until the budget is
    spent and reports its rate, thread count and sample"""
    tf, threads, sample = bench.oracle_sample(seconds_budget=0.2)
    assert tf > 0 and threads >= 1
    assert "23 ResNet-50 layers" in sample and "image" in sample
