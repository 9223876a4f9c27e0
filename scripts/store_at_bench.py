"""store_at measurement (NEXT 1): the BERT-base FC GEMMs of config 3
(M = 8192 tokens) with the bias attached to the weight columns
(alt_matmul_store_at, Z stored [N, K + 8]: column n then bias[n]) against the
same GEMM with a separate fp32 bias vector (alt_matmul, B stored [N, K]).
CUDA events on the launching stream, 10 warm-up + 100 timed launches each,
operands L2-warm (A is 12.6-50 MB, the question is the epilogue, not HBM).
Also times alt_store_at itself (a one-off weight transform).  One JSON line
per shape."""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/", 2)[0])
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth  # noqa: E402


def timed(fn, iters=100, warm=10):
    for _ in range(warm):
        fn()
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(s)
    for _ in range(iters):
        fn()
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / iters  # us


def main():
    dt = torch.bfloat16
    M = 8192
    for (K, N) in [(768, 2304), (768, 768), (768, 3072), (3072, 768)]:
        A = synth.activations("sab_A", (M, K)).to(dt).cuda()
        B = synth.weights("sab_B", (K, N)).to(dt)
        bias = synth.bn_bias("sab_b", N)
        La, Lc = alt.Layout((M, K), []), alt.Layout((M, N), [])
        Lbt = alt.Layout((K, N), [("reorder", [1, 0])])
        bt = B.t().contiguous().cuda()          # B stored [N, K]
        Lb = alt.Layout((K, N), [])
        Lz = alt.Layout((K + 1, N), [("reorder", [1, 0]), ("pad", 1, 0, 7)])
        z = torch.empty(Lz.phys_shape, dtype=dt, device="cuda")
        bd, bb = B.cuda(), bias.to(dt).cuda()
        c0 = torch.empty((M, N), dtype=dt, device="cuda")
        c1 = torch.empty((M, N), dtype=dt, device="cuda")
        bias_f32 = bias.to(dt).float().cuda()   # same (bf16-rounded) bias values
        t_store = timed(lambda: alt.store_at(Lb, bd, bb, 0, Lz, z))
        t_sep = timed(lambda: alt.matmul(M, N, K, La, A, Lbt, bt, Lc, c0, bias=bias_f32))
        p_sep = alt.last_plan()
        t_att = timed(lambda: alt.matmul_store_at(M, N, K, La, A, Lz, z, Lc, c1))
        p_att = alt.last_plan()
        # row-pitch study: separate bias with B rows padded like Z's, and Z
        # rows padded to a 128-byte multiple (bias at the start of a line)
        Lbp = alt.Layout((K, N), [("reorder", [1, 0]), ("pad", 1, 0, 8)])
        bp = torch.empty(Lbp.phys_shape, dtype=dt, device="cuda")
        alt.relayout(Lb, bd, Lbp, bp)
        t_sep_pad8 = timed(lambda: alt.matmul(M, N, K, La, A, Lbp, bp, Lc, c0, bias=bias_f32))
        Lz64 = alt.Layout((K + 1, N), [("reorder", [1, 0]), ("pad", 1, 0, 63)])
        z64 = torch.empty(Lz64.phys_shape, dtype=dt, device="cuda")
        alt.store_at(Lb, bd, bb, 0, Lz64, z64)
        c2 = torch.empty((M, N), dtype=dt, device="cuda")
        t_att64 = timed(lambda: alt.matmul_store_at(M, N, K, La, A, Lz64, z64, Lc, c2))
        torch.cuda.synchronize()
        same = bool(torch.equal(c0, c1)) and bool(torch.equal(c0, c2))
        fl = 2.0 * M * N * K
        print(json.dumps({"M": M, "N": N, "K": K, "separate_bias_us": round(t_sep, 2),
                          "attached_bias_us": round(t_att, 2),
                          "separate_bias_rows_k8_us": round(t_sep_pad8, 2),
                          "attached_bias_rows_k64_us": round(t_att64, 2),
                          "separate_tflops": round(fl / t_sep / 1e6, 1),
                          "attached_tflops": round(fl / t_att / 1e6, 1),
                          "store_at_us": round(t_store, 2), "bitwise_equal": same,
                          "path_sep": p_sep["path"], "path_att": p_att["path"],
                          "block_n": [p_sep.get("block_n"), p_att.get("block_n")]}), flush=True)


if __name__ == "__main__":
    main()
