"""Diagnostics: compress + decompress one config at block length L (warm-up
call first), for ncu captures of the L-specific kernels.
    python tools/run_L.py --L 8 --config c3_hacc --rel 1e-3 [--reps 2]"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangd0lc23_b200 as cz, synth
ap = argparse.ArgumentParser()
ap.add_argument("--L", type=int, default=8)
ap.add_argument("--config", default="c3_hacc")
ap.add_argument("--field", default=None)
ap.add_argument("--rel", type=float, default=1e-3)
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
x = synth.field_for_config(a.config, device="cuda", field=a.field)
mm = torch.stack([x.min(), x.max()])
for _ in range(a.reps):
    out, nb = cz.compress_minmax(x, a.rel, mm, block_len=a.L)
    y = cz.decompress(out, x.numel(), in_bytes=int(nb.item()), block_len=a.L)
torch.cuda.synchronize()
print("status", cz.last_status(), "CR", 4 * x.numel() / int(nb.item()))
