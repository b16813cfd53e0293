import sys, os; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, oracle, paper_conf_sc_huangd0lc23_b200 as cz
n=2; rng=np.random.default_rng(n); x=np.cumsum(rng.standard_normal(n)).astype(np.float32)
for Lb in (32,64,128):
    out, nb = cz.compress(torch.from_numpy(x).cuda(), 1e-3, "rel", block_len=Lb)
    torch.cuda.synchronize()
    s = out[: int(nb.item())].cpu().numpy()
    st, so = oracle.compress_L(x, 1e-3, oracle.REL, Lb)
    print(Lb, s.size, so.size, "F", s[32:36], so[32:36], "payload", np.frombuffer(s[24:32].tobytes(), np.uint64), np.frombuffer(so[24:32].tobytes(), np.uint64))
    print(" gpu", s[48:].view(np.uint32) if s.size > 48 else None)
    print(" ora", so[48:].view(np.uint32))
