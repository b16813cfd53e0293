"""One REL round trip on the HACC-shaped 1.12 GB field after one warm-up
(diagnostics; GPU) -- for `ncu -s 3 -c 3` captures of the large-field kernels:
    ncu --set full -k regex:"range_kernel|compress_kernel|decompress_kernel" -s 3 -c 3 \\
        -o gpurun_out/prof_large python tools/large_field_run.py
"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

x = synth.field_for_config("c3_hacc", device="cuda")
ws = cz.Workspace(x.numel())
for _ in range(2):
    out, nb = cz.compress(x, 1e-3, "rel", ws=ws)
    y = cz.decompress(out, x.numel(), ws=ws)
torch.cuda.synchronize()
assert cz.last_status(ws) == cz.OK
print("ok", int(nb.item()))
