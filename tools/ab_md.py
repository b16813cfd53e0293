"""A/B timing of the multi-dimensional Lorenzo kernels (R18) across library
variants (diagnostics; GPU): compress_md / decompress_md on a Hurricane-U
shaped (100, 500, 500) field and the NYX-shaped 512^3 field, L2 flushed,
ABS bound from the field's range (no range kernel), median of --rounds.
    python tools/ab_md.py lib1.so lib2.so ... [--rounds 7]"""
import argparse, ctypes as C, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch


def load(path):
    h = C.CDLL(path)
    sz, vp, i32, f32 = C.c_size_t, C.c_void_p, C.c_int, C.c_float
    h.cuszp_compress_md.argtypes = [vp, sz, sz, sz, i32, f32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_decompress_md.argtypes = [vp, sz, vp, sz, sz, sz, i32, vp, sz, vp]
    h.cuszp_max_compressed_bytes_md.argtypes = [sz, sz, sz, i32]; h.cuszp_max_compressed_bytes_md.restype = sz
    h.cuszp_workspace_bytes_md.argtypes = [sz, sz, sz, i32]; h.cuszp_workspace_bytes_md.restype = sz
    return h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("libs", nargs="+")
    ap.add_argument("--rounds", type=int, default=7)
    a = ap.parse_args()
    import synth
    libs = [load(p) for p in a.libs]
    fl = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    sp = torch.cuda.current_stream().cuda_stream
    fields = {"hurricane_U": synth.field_for_config("c2_hurricane", device="cuda", field="U").reshape(100, 500, 500),
              "nyx": synth.field_for_config("c4_nyx", device="cuda").reshape(512, 512, 512)}
    for name, x in fields.items():
        nz, ny, nx = x.shape
        eb = float(x.max() - x.min()) * 1e-3
        for dims in (2, 3):
            cap = max(l.cuszp_max_compressed_bytes_md(nz, ny, nx, dims) for l in libs)
            wsb = max(l.cuszp_workspace_bytes_md(nz, ny, nx, dims) for l in libs)
            out = torch.empty(cap, dtype=torch.uint8, device="cuda")
            ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
            ob = torch.zeros(1, dtype=torch.int64, device="cuda")
            y = torch.empty_like(x)
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            res = {i: ([], []) for i in range(len(libs))}
            ref = None
            for r in range(a.rounds + 2):
                for i, h in enumerate(libs):
                    fl.zero_(); ev[0].record()
                    h.cuszp_compress_md(x.data_ptr(), nz, ny, nx, dims, eb, 0, out.data_ptr(), cap, ob.data_ptr(),
                                        ws.data_ptr(), wsb, sp)
                    ev[1].record(); fl.zero_(); ev[2].record()
                    h.cuszp_decompress_md(out.data_ptr(), cap, y.data_ptr(), nz, ny, nx, dims, ws.data_ptr(), wsb, sp)
                    ev[3].record()
                    torch.cuda.synchronize()
                    dg = (int(ob.item()), float(y.double().sum()))
                    ref = ref or dg
                    assert dg == ref, (a.libs[i], dg, ref)
                    if r >= 2:
                        res[i][0].append(ev[0].elapsed_time(ev[1]) * 1e3)
                        res[i][1].append(ev[2].elapsed_time(ev[3]) * 1e3)
            gb = x.numel() * 4 / 1e9
            print(f"== {name} dims={dims} CR={x.numel() * 4 / ref[0]:.2f}")
            for i, p in enumerate(a.libs):
                c, d = np.median(res[i][0]), np.median(res[i][1])
                print(f"  {os.path.basename(p):24s} compress {c:8.1f} us ({gb / c * 1e6:7.1f} GB/s)  "
                      f"decompress {d:8.1f} us ({gb / d * 1e6:7.1f} GB/s)")


if __name__ == "__main__":
    main()
