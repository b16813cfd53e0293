"""A/B timing of cuszp_quality across library variants (diagnostics; GPU).

    python tools/qbench.py lib1.so lib2.so ... [--n 25000000] [--rounds 7]
"""
import argparse, ctypes as C, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch

ap = argparse.ArgumentParser()
ap.add_argument("libs", nargs="+")
ap.add_argument("--n", type=int, default=25_000_000)
ap.add_argument("--rounds", type=int, default=7)
a = ap.parse_args()
dev = torch.device("cuda", 0)
x = torch.randn(a.n, device=dev) * 30 + 250
y = x + 1e-3 * torch.randn(a.n, device=dev)
q = torch.empty(14, dtype=torch.float64, device=dev)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
sink = torch.empty(1, dtype=torch.int64, device=dev)
sp = torch.cuda.current_stream().cuda_stream
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
libs = []
for p in a.libs:
    h = C.CDLL(p)
    h.cuszp_quality_workspace_bytes.restype = C.c_size_t
    h.cuszp_quality.argtypes = [C.c_void_p, C.c_void_p, C.c_size_t, C.c_double, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p]
    ws = torch.zeros(h.cuszp_quality_workspace_bytes(), dtype=torch.uint8, device=dev)
    libs.append((p, h, ws))
res = {p: [] for p, _, _ in libs}
ref = None
for r in range(a.rounds + 1):
    for p, h, ws in libs:
        flush.zero_(); sink.copy_(flush.view(torch.int64).sum())
        ev[0].record()
        assert h.cuszp_quality(x.data_ptr(), y.data_ptr(), a.n, 1e-3, q.data_ptr(), ws.data_ptr(), ws.numel(), sp) == 0
        ev[1].record()
        torch.cuda.synchronize()
        v = q.cpu().numpy().copy()
        if ref is None: ref = v
        assert np.array_equal(v[[0, 1, 2, 3, 4, 5]], ref[[0, 1, 2, 3, 4, 5]]), (p, v, ref)
        if r: res[p].append(ev[0].elapsed_time(ev[1]) * 1e3)
for p, t in res.items():
    print(f"{os.path.basename(p):30s} quality {np.median(t):7.1f} us  = {8 * a.n / np.median(t) / 1e3:7.1f} GB/s")
