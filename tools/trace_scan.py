"""Per-tile timeline of the two scan kernels (diagnostics; needs a GPU).

    python tools/trace_scan.py [--lib path/to/libcuszp_variant.so] [--config c2_hurricane]

Needs a library built with -DCUSZP_TRACE (the production build compiles the
compute-warp trace points out: a lane-0 branch in the encode loop costs ~6 %):
    python tools/build_variants.py trace:CUSZP_TRACE
    python tools/trace_scan.py --lib build_variants/trace.so

Installs a trace buffer (cuszp_debug_set_trace), runs range + compress +
decompress on one field and prints, per kernel, the distribution of the
per-tile phases recorded with %globaltimer:
  slot 0 ticket taken, 1 compute start, 2 aggregate published,
  3 look-back start, 4 prefix resolved, 5 windows walked, 6 spins, 7 data in shared memory
"""
from __future__ import annotations

import argparse
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402


def load(path):
    h = C.CDLL(path)
    sz, vp, i32, f32 = C.c_size_t, C.c_void_p, C.c_int, C.c_float
    h.cuszp_range.argtypes = [vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_minmax.argtypes = [vp, sz, f32, vp, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_decompress.argtypes = [vp, sz, vp, sz, vp, sz, vp]
    h.cuszp_workspace_bytes.argtypes = [sz]
    h.cuszp_workspace_bytes.restype = sz
    h.cuszp_max_compressed_bytes.argtypes = [sz]
    h.cuszp_max_compressed_bytes.restype = sz
    h.cuszp_debug_set_trace.argtypes = [vp]
    h.cuszp_compress_minmax_L.argtypes = [vp, sz, f32, vp, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_max_compressed_bytes_L.argtypes = [sz, i32]
    h.cuszp_max_compressed_bytes_L.restype = sz
    return h


def pct(a, qs=(10, 50, 90, 99)):
    return " ".join(f"p{q}={np.percentile(a, q):8.2f}" for q in qs)


def report(name, tr, total_ns):
    t0 = tr[:, 0].min()
    ticket = (tr[:, 0] - t0) / 1e3
    landed = (tr[:, 1] - t0) / 1e3
    agg = (tr[:, 2] - t0) / 1e3
    lb0 = (tr[:, 3] - t0) / 1e3
    pfx = (tr[:, 4] - t0) / 1e3
    print(f"== {name}: {tr.shape[0]} tiles, kernel span {total_ns / 1e3:.1f} us (first ticket .. last prefix "
          f"{(tr[:, 4].max() - t0) / 1e3:.1f} us)")
    print(f"  TMA issue -> landed     (us) {pct((tr[:, 7] - t0) / 1e3 - ticket)}")
    print(f"  landed -> compute start (us) {pct(landed - (tr[:, 7] - t0) / 1e3)}  (meta-slot wait)")
    print(f"  landed -> aggregate     (us) {pct(agg - landed)}")
    print(f"  aggregate -> lb start   (us) {pct(lb0 - agg)}")
    print(f"  look-back duration      (us) {pct(pfx - lb0)}")
    print(f"  ticket -> prefix        (us) {pct(pfx - ticket)}")
    print(f"  windows {pct(tr[:, 5])}   spins {pct(tr[:, 6])}")
    print(f"  windows mean {tr[:, 5].mean():.2f} max {tr[:, 5].max()}   spins mean {tr[:, 6].mean():.2f} max {tr[:, 6].max()}"
          f"  (sum {tr[:, 6].sum()})")
    # lag: at each prefix time, how many tiles with smaller index had no aggregate yet
    order = np.argsort(tr[:, 2])
    print(f"  aggregate order vs ticket order: mean |rank diff| = {np.abs(np.argsort(order) - np.arange(len(order))).mean():.1f}")
    # throughput over time (tiles resolved per 10 us)
    bins = np.arange(0, (tr[:, 4].max() - t0) / 1e3 + 10, 10)
    hist, _ = np.histogram(pfx, bins)
    print("  prefixes per 10 us:", " ".join(str(v) for v in hist))


def report_d(tr):
    t0 = tr[:, 0].min()
    rel = lambda k: (tr[:, k] - t0) / 1e3
    print(f"== decompress: {tr.shape[0]} tiles, first ticket .. last done {(tr[:, 5].max() - t0) / 1e3:.1f} us")
    names = ["ticket", "F+A", "prefix", "TMA issued", "1st pickup", "last done"]
    for a, b in zip(range(5), range(1, 6)):
        print(f"  {names[a]:>10s} -> {names[b]:<10s} (us) {pct(rel(b) - rel(a))}")
    print(f"  windows {pct(tr[:, 6] >> 32)}  spins {pct(tr[:, 6] & 0xffffffff)}")
    bins = np.arange(0, rel(5).max() + 10, 10)
    print("  tiles done per 10 us:", " ".join(str(v) for v in np.histogram(rel(5), bins)[0]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lib", default=os.path.join(ROOT, "paper_conf_sc_huangd0lc23_b200", "libcuszp.so"))
    ap.add_argument("--config", default="c2_hurricane")
    ap.add_argument("--rel", type=float, default=1e-2)
    ap.add_argument("--field", default=None)
    ap.add_argument("--L", type=int, default=32, help="block length; L != 32 traces compression only")
    a = ap.parse_args()
    import synth

    h = load(a.lib)
    dev = torch.device("cuda", 0)
    x = synth.field_for_config(a.config, device=dev, field=a.field)
    n = x.numel()
    nt = ((n + 31) // 32 + 127) // 128
    ws = torch.zeros(h.cuszp_workspace_bytes(n), dtype=torch.uint8, device=dev)
    cap = h.cuszp_max_compressed_bytes_L(n, a.L)
    out = torch.empty(cap, dtype=torch.uint8, device=dev)
    ob = torch.zeros(1, dtype=torch.int64, device=dev)
    mm = torch.empty(2, dtype=torch.float32, device=dev)
    y = torch.empty(n, dtype=torch.float32, device=dev)
    trace = torch.zeros(nt * 24, dtype=torch.int64, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    sp = torch.cuda.current_stream().cuda_stream
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    for it in range(4):
        traced = it == 3
        if traced:
            trace.zero_()
            trace[nt * 8: nt * 8 + 4] = (1 << 62)          # atomicMin slots
            trace[nt * 8 + 2] = 0
        h.cuszp_debug_set_trace(trace.data_ptr() if traced else None)
        flush.zero_()
        h.cuszp_range(x.data_ptr(), n, mm.data_ptr(), ws.data_ptr(), ws.numel(), sp)
        ev[0].record()
        h.cuszp_compress_minmax_L(x.data_ptr(), n, a.rel, mm.data_ptr(), 1, a.L, out.data_ptr(), cap, ob.data_ptr(),
                                  ws.data_ptr(), ws.numel(), sp)
        ev[1].record()
        if traced:
            torch.cuda.synchronize()
            trc = trace[: nt * 8].view(nt, 8).cpu().numpy().astype(np.int64)
            kk = trace[nt * 8: nt * 8 + 4].cpu().numpy().astype(np.int64)
            t0c = trc[:, 0].min()
            print(f"compress kernel points rel. first ticket (us): first entry {(kk[0] - t0c) / 1e3:.2f}, "
                  f"past pdl_wait {(kk[1] - t0c) / 1e3:.2f}, past prologue {(kk[3] - t0c) / 1e3:.2f}, "
                  f"last prefix {(trc[:, 4].max() - t0c) / 1e3:.2f}, finish {(kk[2] - t0c) / 1e3:.2f}")
            rec = trace[nt * 8: nt * 16].view(nt, 8).cpu().numpy().astype(np.int64)[:, 4:]
            if rec[1:, 0].any():
                # in-place kernels: recycler / writer points (slots 4-7 of region 2)
                sel = slice(1, None)
                agg_t = trc[sel, 2]
                print("in-place compress, per tile (us):")
                print(f"  aggregate -> recycler picks up  {pct((rec[sel, 0] - agg_t) / 1e3)}")
                print(f"  picked up -> room/slot ok      {pct((rec[sel, 1] - rec[sel, 0]) / 1e3)}")
                print(f"  room ok -> parked (stage free) {pct((rec[sel, 2] - rec[sel, 1]) / 1e3)}")
                print(f"  prefix -> released             {pct((rec[sel, 3] - trc[sel, 4]) / 1e3)}")
                print(f"  parked -> released             {pct((rec[sel, 3] - rec[sel, 2]) / 1e3)}")
            trace.zero_()
            trace[: nt * 8].view(nt, 8)[:, 4] = (1 << 62)
        if a.L != 32:
            continue
        flush.zero_()
        ev[2].record()
        h.cuszp_decompress(out.data_ptr(), cap, y.data_ptr(), n, ws.data_ptr(), ws.numel(), sp)
        torch.cuda.synchronize()
    h.cuszp_debug_set_trace(None)
    if a.L != 32:
        S = int(ob.item())
        print(f"n={n} tiles={nt} S={S} CR={4 * n / S:.2f} L={a.L}  compress {ev[0].elapsed_time(ev[1]) * 1e3:.1f} us")
        report("compress", trc, ev[0].elapsed_time(ev[1]) * 1e6)
        return
    trd = trace[: nt * 8].view(nt, 8).cpu().numpy().astype(np.int64)
    pw = trace[nt * 8:nt * 16].view(nt, 8).cpu().numpy().astype(np.int64)
    pk = trace[nt * 16:].view(nt, 8).cpu().numpy().astype(np.int64)
    busy = (pw - pk) / 1e3
    print("decompress per-warp tile compute (pickup -> done, us):", pct(busy.ravel()))
    # per CTA (slot 7) and warp: idle gap between finishing one tile and picking up the next
    cta = trd[:, 7]
    gaps, waits = [], []
    for c in np.unique(cta):
        idx = np.nonzero(cta == c)[0]
        idx = idx[np.argsort(pk[idx, 0])]
        for wv in range(8):
            g = (pk[idx[1:], wv] - pw[idx[:-1], wv]) / 1e3
            gaps.append(g)
            waits.append((pk[idx[1:], wv] - np.maximum(pw[idx[:-1], wv], trd[idx[1:], 3])) / 1e3)
    gaps = np.concatenate(gaps)
    print("decompress per-warp gap done(k) -> pickup(k+1) (us):", pct(gaps), f" mean {gaps.mean():.2f}")
    print("   of which after the next tile's TMA was issued (us):", pct(np.concatenate(waits)))
    span = (pw.max() - pk.min()) / 1e3
    print(f"   warp busy fraction: {busy.sum() / (span * 8 * len(np.unique(cta))):.2f}")
    # per warp slot, consecutive tiles of the same CTA are not identifiable; use the
    # distribution of each warp's pickup relative to the tile's TMA issue instead
    wait = (pk - trd_issue[:, None]) / 1e3 if False else None
    last = np.argmax(pw, axis=1)
    spread = (pw.max(axis=1) - pw.min(axis=1)) / 1e3
    print("decompress: which compute warp finishes a tile last:", np.bincount(last, minlength=8).tolist(),
          " spread first..last warp (us):", pct(spread))
    S = int(ob.item())
    print(f"n={n} tiles={nt} S={S} CR={4 * n / S:.2f}  compress {ev[0].elapsed_time(ev[1]) * 1e3:.1f} us")
    report("compress", trc, ev[0].elapsed_time(ev[1]) * 1e6)
    report_d(trd)


if __name__ == "__main__":
    main()
