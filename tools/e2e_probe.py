"""Where the e2e time of one c3 round trip goes (diagnostics; GPU): copy-engine
H2D / D2H of the field, the device kernels, and the whole host-async calls
(the difference is the SM copy of the stream over mapped memory)."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

cfg = sys.argv[1] if len(sys.argv) > 1 else "c3_hacc"
x = synth.field_for_config(cfg, device="cuda")
n = x.numel()
cap = cz.max_compressed_bytes(n)
h_in = x.cpu().pin_memory()
h_out = torch.zeros(cap, dtype=torch.uint8).pin_memory()
h_len = torch.zeros(1, dtype=torch.int64).pin_memory()
h_y = torch.empty(n).pin_memory()
d_in = torch.empty(n, device="cuda"); d_out = torch.empty(cap, dtype=torch.uint8, device="cuda")
d_y = torch.empty(n, device="cuda"); ws = cz.Workspace(n)
s = torch.cuda.current_stream()


def t(fn, reps=3):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


r = {}
r["h2d_field"] = t(lambda: d_in.copy_(h_in, non_blocking=True))
r["d2h_field"] = t(lambda: h_y.copy_(d_y, non_blocking=True))
r["compress_dev"] = t(lambda: cz.compress(d_in, 1e-3, "rel", out=d_out, ws=ws))
S = int(cz.compress(d_in, 1e-3, "rel", out=d_out, ws=ws)[1].item())
r["decompress_dev"] = t(lambda: cz.decompress(d_out, n, out=d_y, in_bytes=S, ws=ws))
r["compress_host_async"] = t(lambda: cz.compress_host_async(h_in, 1e-3, "rel", h_out, h_len, d_in, d_out, ws))
r["decompress_host_async"] = t(lambda: cz.decompress_host_async(h_out, h_y, d_out, d_y, ws))
r["mapped_d2h_stream"] = r["compress_host_async"] - r["h2d_field"] - r["compress_dev"]
r["mapped_h2d_stream"] = r["decompress_host_async"] - r["d2h_field"] - r["decompress_dev"]
print(f"n={n} S={S} ({S / 1e9:.3f} GB)")
for k, v in r.items():
    b = 4 * n if "field" in k else S if "stream" in k else None
    print(f"{k:24s} {v * 1e3:8.2f} ms" + (f"  {b / v / 1e9:6.1f} GB/s" if b else ""))
