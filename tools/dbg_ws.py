import sys, os; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, paper_conf_sc_huangd0lc23_b200 as cz
def ctrl(tag):
    ws = cz._workspace(1, torch.device("cuda", 0), None)
    torch.cuda.synchronize()
    w = ws.buf[:128].cpu().view(torch.int32).numpy()
    print(tag, "epoch", w[0], "ticket", w[1], "exit", w[2], "acc", w[3], "last", w[4], "rmax", hex(w[5] & 0xffffffff), "rmin", hex(w[6] & 0xffffffff), "rexit", w[7], "mm", ws.buf[32:40].cpu().view(torch.float32).numpy())
rng = np.random.default_rng(5)
xf = torch.from_numpy(rng.standard_normal(70_000).astype(np.float32)).cuda()
for Lb in (64, 128):
    for n in [2, 31, 64, 65, 129, 4096, 4097, 100_003, 1 << 20]:
        r = np.random.default_rng(n)
        x = np.cumsum(r.standard_normal(n)).astype(np.float32); x[n // 3: n // 2] = 0.0
        out, nb = cz.compress(torch.from_numpy(x).cuda(), 1e-3, "rel", block_len=Lb)
        torch.cuda.synchronize()
        s = out[: int(nb.item())]
        y = cz.decompress(out, n, in_bytes=s.numel(), block_len=Lb)
        out2, nb2 = cz.compress(xf, 1e-3, "rel")
        torch.cuda.synchronize()
        st = cz.read_header(out2)["status"]
        if st != 0:
            print("BROKEN after", Lb, n); ctrl("state"); sys.exit(0)
print("no failure")
