"""Diagnostics: compress_md + decompress_md of a Hurricane-U-shaped field
(100 x 500 x 500) with the 2D or 3D predictor (two calls; for ncu captures).
    python tools/run_md.py --dims 3 [--reps 2]"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangd0lc23_b200 as cz, synth
ap = argparse.ArgumentParser()
ap.add_argument("--dims", type=int, default=3)
ap.add_argument("--rel", type=float, default=1e-3)
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
x = synth.field_for_config("c2_hurricane", device="cuda", field="U").reshape(100, 500, 500)
for _ in range(a.reps):
    out, nb = cz.compress_md(x, a.rel, "rel", dims=a.dims)
    y = cz.decompress_md(out, tuple(x.shape), a.dims, in_bytes=int(nb.item()))
torch.cuda.synchronize()
print("CR", 4 * x.numel() / int(nb.item()))
