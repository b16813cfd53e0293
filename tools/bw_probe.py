"""Achievable HBM bandwidth for the bench's array size (diagnostics; GPU).

    python tools/bw_probe.py [--mb 100]

Times, with a clean L2 flush before each launch (CUDA events): torch sum
(read), clone (read+write), fill (write), and our range kernel, on an
array of the given size -- the ceilings the three kernels are compared to.
"""
import argparse, ctypes as C, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch

ap = argparse.ArgumentParser()
ap.add_argument("--mb", type=float, default=100)
ap.add_argument("--lib", default=os.path.join(ROOT, "paper_conf_sc_huangd0lc23_b200", "libcuszp.so"))
a = ap.parse_args()
dev = torch.device("cuda", 0)
n = int(a.mb * 1e6 / 4)
x = torch.randn(n, device=dev)
y = torch.empty_like(x)
fb = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
sink = torch.empty(1, dtype=torch.int64, device=dev)
h = C.CDLL(a.lib)
h.cuszp_workspace_bytes.restype = C.c_size_t
ws = torch.zeros(h.cuszp_workspace_bytes(C.c_size_t(n)), dtype=torch.uint8, device=dev)
mm = torch.empty(2, device=dev)
sp = torch.cuda.current_stream().cuda_stream


def flush():
    fb.zero_(); sink.copy_(fb.view(torch.int64).sum())


def t(fn, reps=9):
    ts = []
    for _ in range(reps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


B = 4 * n
for name, fn, nbytes in [
    ("torch sum (read)", lambda: x.sum(), B),
    ("torch aminmax (read)", lambda: torch.aminmax(x), B),
    ("clone (read+write)", lambda: y.copy_(x), 2 * B),
    ("fill (write)", lambda: y.fill_(1.0), B),
    ("cuszp_range (read)", lambda: h.cuszp_range(C.c_void_p(x.data_ptr()), C.c_size_t(n), C.c_void_p(mm.data_ptr()),
                                                 C.c_void_p(ws.data_ptr()), C.c_size_t(ws.numel()), C.c_void_p(sp)), B),
]:
    us = t(fn)
    print(f"{name:24s} {us:8.1f} us  {nbytes / us / 1e3:7.1f} GB/s")
