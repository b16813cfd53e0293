"""One warm-up + one measured round trip per library variant on a config,
for ncu captures that compare variants (diagnostics; GPU):
    ncu --metrics ... -k regex:compress_kernel python tools/ncu_ab.py lib1.so lib2.so --config c3_hacc
Launch order per lib: range, compress, decompress (x2)."""
import argparse, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch
from ab import load

ap = argparse.ArgumentParser()
ap.add_argument("libs", nargs="+")
ap.add_argument("--config", default="c3_hacc")
ap.add_argument("--field", default=None)
ap.add_argument("--rel", type=float, default=1e-3)
a = ap.parse_args()
import synth
x = synth.field_for_config(a.config, device="cuda", field=a.field)
n = x.numel()
libs = [load(p) for p in a.libs]
ws = torch.zeros(max(l.cuszp_workspace_bytes(n) for l in libs), dtype=torch.uint8, device="cuda")
cap = max(l.cuszp_max_compressed_bytes(n) for l in libs)
out = torch.empty(cap, dtype=torch.uint8, device="cuda")
ob = torch.zeros(1, dtype=torch.int64, device="cuda")
mm = torch.empty(2, dtype=torch.float32, device="cuda")
y = torch.empty(n, dtype=torch.float32, device="cuda")
sp = torch.cuda.current_stream().cuda_stream
for h in libs:
    ws.zero_()
    for _ in range(2):
        h.cuszp_range(x.data_ptr(), n, mm.data_ptr(), ws.data_ptr(), ws.numel(), sp)
        h.cuszp_compress_minmax(x.data_ptr(), n, a.rel, mm.data_ptr(), 1, out.data_ptr(), cap, ob.data_ptr(),
                                ws.data_ptr(), ws.numel(), sp)
        h.cuszp_decompress(out.data_ptr(), cap, y.data_ptr(), n, ws.data_ptr(), ws.numel(), sp)
    torch.cuda.synchronize()
    print(os.path.basename(a.libs[libs.index(h)]), int(ob.item()))
