import sys, ctypes as C, torch
sys.path.insert(0, '.')
from paper_conf_icpp_0002s22_b200 import lf
L = lf.load(); L.lf_debug_launch_probe.argtypes = [C.c_int, C.c_int, C.c_int, C.c_void_p]
s = torch.cuda.current_stream()
def t(mode, block, steps, reps=50, graph=False):
    fn = lambda: L.lf_debug_launch_probe(mode, block, steps, C.c_void_p(s.cuda_stream))
    for _ in range(5): fn()
    torch.cuda.synchronize()
    if graph:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(reps): fn()
        g.replay(); torch.cuda.synchronize()
        e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        e0.record(); g.replay(); e1.record(); e1.synchronize()
    else:
        e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        e0.record()
        for _ in range(reps): fn()
        e1.record(); e1.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3
for graph in (False, True):
    print("graph" if graph else "eager")
    print(" plain 256:", round(t(0, 256, 0, graph=graph), 2), "us")
    print(" plain 1024:", round(t(0, 1024, 0, graph=graph), 2), "us")
    for blk in (256, 1024):
        for st in (0, 1, 5, 20):
            print(f" coop {blk} syncs={st}:", round(t(1, blk, st, graph=graph), 2), "us")
