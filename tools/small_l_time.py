"""Median compress / decompress times of every block length on the Hurricane U field (100 MB), L2 flushed."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, time, json
import paper_conf_sc_huangd0lc23_b200 as cz, synth
from synth import hurricane_like
x = hurricane_like("U", shape=(100, 500, 500), device="cuda")
res = {}
for Lb in (8, 16, 32, 64, 128):
    out, nb = cz.compress(x, 1e-3, "rel", block_len=Lb)
    y = cz.decompress(out, x.numel(), block_len=Lb)
    torch.cuda.synchronize()
    fl = torch.empty(400 << 20, dtype=torch.uint8, device="cuda")
    tc, td = [], []
    for it in range(8):
        fl.zero_(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); cz.compress(x, 1e-3, "rel", out=out, block_len=Lb); e.record(); torch.cuda.synchronize(); tc.append(s.elapsed_time(e))
        fl.zero_(); s.record(); cz.decompress(out, x.numel(), out=y, block_len=Lb); e.record(); torch.cuda.synchronize(); td.append(s.elapsed_time(e))
    tc, td = sorted(tc[2:])[len(tc[2:])//2], sorted(td[2:])[len(td[2:])//2]
    res[Lb] = dict(cr=x.numel()*4/int(nb.item()), compress_gbs=x.numel()*4/tc/1e6, decompress_gbs=x.numel()*4/td/1e6,
                   compress_ms=tc, decompress_ms=td, status=cz.last_status())
print(json.dumps(res, indent=1))
