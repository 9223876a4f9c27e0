import torch
def timeit(fn, reps=20, graph=True):
    """us per call; graph=True replays `reps` calls captured in a CUDA graph
    (no host launch overhead; consecutive kernels may overlap via PDL)."""
    for _ in range(3): fn()
    torch.cuda.synchronize()
    g = None
    if graph:
        try:
            g = torch.cuda.CUDAGraph()
            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(s), torch.cuda.graph(g, stream=s):
                for _ in range(reps): fn()
            torch.cuda.current_stream().wait_stream(s)
        except Exception:
            g = None
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    if g is not None:
        g.replay()
    else:
        for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3
