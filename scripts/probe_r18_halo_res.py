import sys, torch
sys.path.insert(0, '.')
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as A
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from scripts.exptime import timeit
ch = CH.resnet18(256, torch.device('cuda', 0))
ch.run(); torch.cuda.synchronize()
for i in (2, 3):
    op = ch.ops[i]
    L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
    wl, w, sc, bi = ch.weights[i]
    p = A.conv_params(ch.N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad, L.groups)
    kw = dict(residual=ch.buf[res], residual_l=ch.layouts[res]) if res is not None else {}
    for c in ({'path': 1, 'block_n': 64, 'cta_pair': 2, 'tile_n': 2, 'tile_h': 1, 'tile_w': 64, 'block_k': 1}, ch.cfgs.get(i)):
        try:
            t = timeit(lambda: A.conv2d(p, ch.layouts[src], ch.buf[src], wl, w, ch.layouts[dst], ch.buf[dst], scale=sc, bias=bi, act='relu', cfg=c, pads_zero=True, **kw))
            print(i, L.name, c, round(t, 1), A.last_plan())
        except Exception as e:
            print(i, L.name, c, 'ERR', e)
