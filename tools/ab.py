"""A/B timing of library variants (diagnostics; needs a GPU).

    python tools/ab.py lib1.so lib2.so ... [--rounds 5] [--config c2_hurricane] [--rel 1e-2]

Every round times each variant's range, compress (compress_minmax) and
decompress kernels with CUDA events, L2 flushed before each launch; prints
the median and min per variant.  Variants are interleaved so clock ramps and
box noise hit them alike.
"""
import argparse, ctypes as C, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch


def load(path):
    h = C.CDLL(path)
    sz, vp, i32, f32 = C.c_size_t, C.c_void_p, C.c_int, C.c_float
    h.cuszp_range.argtypes = [vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_minmax.argtypes = [vp, sz, f32, vp, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress.argtypes = [vp, sz, f32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_decompress.argtypes = [vp, sz, vp, sz, vp, sz, vp]
    h.cuszp_workspace_bytes.argtypes = [sz]; h.cuszp_workspace_bytes.restype = sz
    h.cuszp_max_compressed_bytes.argtypes = [sz]; h.cuszp_max_compressed_bytes.restype = sz
    h.cuszp_max_compressed_bytes_L.argtypes = [sz, i32]; h.cuszp_max_compressed_bytes_L.restype = sz
    h.cuszp_compress_minmax_L.argtypes = [vp, sz, f32, vp, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_L.argtypes = [vp, sz, f32, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_decompress_L.argtypes = [vp, sz, vp, sz, i32, vp, sz, vp]
    return h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("libs", nargs="+")
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--config", default="c2_hurricane")
    ap.add_argument("--field", default=None)
    ap.add_argument("--rel", type=float, default=1e-2)
    ap.add_argument("--nocheck", action="store_true")
    ap.add_argument("--L", type=int, default=32, help="block length (8, 16, 32, 64, 128)")
    ap.add_argument("--dirty-flush", action="store_true")
    a = ap.parse_args()
    import synth
    dev = torch.device("cuda", 0)
    x = synth.field_for_config(a.config, device=dev, field=a.field)
    n = x.numel()
    libs = [load(p) for p in a.libs]
    h0 = libs[0]
    ws = torch.zeros(max(l.cuszp_workspace_bytes(n) for l in libs), dtype=torch.uint8, device=dev)
    cap = max(l.cuszp_max_compressed_bytes_L(n, a.L) for l in libs)
    L = a.L
    out = torch.empty(cap, dtype=torch.uint8, device=dev)
    ob = torch.zeros(1, dtype=torch.int64, device=dev)
    mm = torch.empty(2, dtype=torch.float32, device=dev)
    y = torch.empty(n, dtype=torch.float32, device=dev)
    flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    sink = torch.empty(1, dtype=torch.int64, device=dev)

    class _F:
        @staticmethod
        def zero_():
            # write then read 512 MB: L2 ends up holding CLEAN lines of an
            # unrelated buffer (a write-only flush leaves ~126 MB of dirty lines
            # whose write-back would be charged to the next timed kernel)
            flush_buf.zero_()
            if not a.dirty_flush:
                sink.copy_(flush_buf.view(torch.int64).sum())
    flush = _F
    sp = torch.cuda.current_stream().cuda_stream
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
    res = {i: {"range": [], "compress": [], "decompress": [], "rel_chain": [], "rel_call": []} for i in range(len(libs))}
    ref = None
    for r in range(a.rounds + 2):
        for i, h in enumerate(libs):
            ws.zero_()
            flush.zero_(); ev[0].record()
            h.cuszp_range(x.data_ptr(), n, mm.data_ptr(), ws.data_ptr(), ws.numel(), sp); ev[1].record()
            flush.zero_(); ev[2].record()
            h.cuszp_compress_minmax_L(x.data_ptr(), n, a.rel, mm.data_ptr(), 1, L, out.data_ptr(), cap, ob.data_ptr(),
                                      ws.data_ptr(), ws.numel(), sp); ev[3].record()
            flush.zero_(); ev[4].record()
            h.cuszp_decompress_L(out.data_ptr(), cap, y.data_ptr(), n, L, ws.data_ptr(), ws.numel(), sp); ev[5].record()
            # REL chain as the product runs it: flush, range, compress (no flush between)
            flush.zero_(); ev[6].record()
            h.cuszp_range(x.data_ptr(), n, mm.data_ptr(), ws.data_ptr(), ws.numel(), sp)
            h.cuszp_compress_minmax_L(x.data_ptr(), n, a.rel, mm.data_ptr(), 1, L, out.data_ptr(), cap, ob.data_ptr(),
                                      ws.data_ptr(), ws.numel(), sp); ev[7].record()
            # REL as one call (range + compress; the library may overlap them)
            flush.zero_(); ev[8].record()
            h.cuszp_compress_L(x.data_ptr(), n, a.rel, 1, L, out.data_ptr(), cap, ob.data_ptr(), ws.data_ptr(),
                               ws.numel(), sp); ev[9].record()
            torch.cuda.synchronize()
            S = int(ob.item())
            digest = (S, float(y[:1000].sum()), float(y[-1000:].sum()))
            if ref is None: ref = digest
            if not a.nocheck: assert digest == ref, (a.libs[i], digest, ref)
            if r >= 2:
                res[i]["range"].append(ev[0].elapsed_time(ev[1]) * 1e3)
                res[i]["compress"].append(ev[2].elapsed_time(ev[3]) * 1e3)
                res[i]["decompress"].append(ev[4].elapsed_time(ev[5]) * 1e3)
                res[i]["rel_chain"].append(ev[6].elapsed_time(ev[7]) * 1e3)
                res[i]["rel_call"].append(ev[8].elapsed_time(ev[9]) * 1e3)
    print(f"n={n} S={ref[0]} CR={4 * n / ref[0]:.2f}  (us: median / min)")
    occ = (C.c_int * 4)()
    for p_, h in zip(a.libs, libs):
        if hasattr(h, "cuszp_debug_occupancy") and h.cuszp_debug_occupancy(occ) == 0:
            print(f"   {os.path.basename(p_):38s} SMs {occ[0]}  CTAs/SM: compress {occ[1]} decompress {occ[2]} range {occ[3]}")
    for i, p in enumerate(a.libs):
        d = res[i]
        print(f"{os.path.basename(p):40s} range {np.median(d['range']):7.1f}/{min(d['range']):7.1f}  "
              f"compress {np.median(d['compress']):7.1f}/{min(d['compress']):7.1f}  "
              f"decompress {np.median(d['decompress']):7.1f}/{min(d['decompress']):7.1f}  "
              f"range+compress {np.median(d['rel_chain']):7.1f}  REL call {np.median(d['rel_call']):7.1f}")


if __name__ == "__main__":
    main()
