"""Tune cache (SURVEY §5 "checkpoint / resume"): alt_tune results keyed by
(op, shape, per-GPU batch, dtype, GPU name), stored as JSON lines in
tune_cache.jsonl at the repo root, so chains and benches re-run without
re-tuning."""
from __future__ import annotations

import json
import os

_PATH = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tune_cache.jsonl")
_cache = None


def key(op: str, L, N: int, dtype: str = "bf16") -> str:
    return f"{op}|N{N}|C{L.C}|H{L.H}|W{L.W}|K{L.K}|R{L.R}|S{L.S}|s{L.stride}|p{L.pad}|g{L.groups}|{dtype}"


def _load():
    global _cache
    if _cache is None:
        _cache = {}
        if os.path.exists(_PATH):
            for line in open(_PATH):
                line = line.strip()
                if line:
                    e = json.loads(line)
                    _cache[e["key"]] = e
    return _cache


def _tup(prims):
    return [tuple(p) if p[0] not in ("split", "reorder") else
            ((p[0], p[1], list(p[2])) if p[0] == "split" else (p[0], list(p[1]))) for p in prims]


def lookup(op: str, L, N: int, dtype: str = "bf16"):
    e = _load().get(key(op, L, N, dtype))
    if e is None:
        return None
    return {"x": _tup(e["x"]), "w": _tup(e["w"]), "y": _tup(e["y"]), "cfg": e["cfg"],
            "us": e.get("us")}


def store(op: str, L, N: int, result: dict, dtype: str = "bf16"):
    c = _load()
    e = {"key": key(op, L, N, dtype), "x": result["x"], "w": result["w"], "y": result["y"],
         "cfg": result["cfg"], "us": result.get("best_us")}
    c[e["key"]] = e
    with open(_PATH, "w") as f:
        for v in c.values():
            f.write(json.dumps(v) + "\n")


def gemm_key(M: int, N: int, K: int, dtype: str = "bf16") -> str:
    return f"matmul|M{M}|N{N}|K{K}|{dtype}"


def lookup_gemm(M: int, N: int, K: int, dtype: str = "bf16"):
    """kernel configuration for a GEMM on the bench's tiled layouts, or None"""
    e = _load().get(gemm_key(M, N, K, dtype))
    return None if e is None else e["cfg"]


def store_gemm(M: int, N: int, K: int, cfg: dict, us: float, dtype: str = "bf16"):
    c = _load()
    c[gemm_key(M, N, K, dtype)] = {"key": gemm_key(M, N, K, dtype), "cfg": cfg, "us": us}
    with open(_PATH, "w") as f:
        for v in c.values():
            f.write(json.dumps(v) + "\n")
