#!/usr/bin/env python
"""bench.py -- throughput of the cuSZp hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N --steps K --warmup W] [--impl ours|reference]
                    [--config c2_hurricane|c1_smooth1d|c3_hacc|c4_nyx|c5_rtm]

A STEP is one pass of the whole hot path over one
batch of synthetic input: for every field of the config and every REL error
bound it names, value range (a1) -> fused compression (a2..a8) -> fused
decompression (a9..a12), all through the C ABI.  The default workload is
BASELINE configs[1]: three Hurricane-shaped 100x500x500 fp32 fields (U,
QCLOUD, TC) at REL 1e-2, 1e-3, 1e-4 -> 9 round trips, 900 MB of fp32 input
per step per GPU.

Timing: the L2 (126 MB) is flushed (a 512 MB write + read, untimed) before every
round trip; each round trip is bracketed by CUDA events on the launching
stream; a step's time is the sum of its round trips' device time.  W warm-up
steps, then K timed steps between barrier + synchronize; max over ranks.
Multi-GPU (torchrun): weak scaling -- every rank compresses its own fields
with the GLOBAL REL range (NCCL all-gather of (min,max)) and all-gathers the
compressed byte counts to build the container header (paper_conf_sc_
huangd0lc23_b200.dist).

--impl reference runs the CPU oracle (oracle/, single thread) on a bounded
sample of the same config -- the tier's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

PAPER_A100 = {"compress_mean_gbs": 93.63, "decompress_mean_gbs": 120.04,
              "source": "PAPER.md P:961-962 (A100 40GB, real SDRBench data, REL 1E-1..1E-4)"}
FALLBACK_HBM_GBS = 6650.0


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="c2_hurricane")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-large", action="store_true", help="skip the 1.12 GB HACC-shaped context measurement")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=10.0)
    return p.parse_args()


# ------------------------------------------------------------------ helpers

def peak_hbm():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """SM clock + clock-event (throttle) reasons polled through NVML every
    ~2 ms from a thread while the timed region runs (the region lasts tens of
    ms, too short for nvidia-smi's 100 ms sampling).  Falls back to
    nvidia-smi when NVML is unavailable."""
    NAMES = {"hw_slowdown": "nvmlClocksEventReasonHwSlowdown",
             "hw_thermal_slowdown": "nvmlClocksEventReasonHwThermalSlowdown",
             "sw_thermal_slowdown": "nvmlClocksEventReasonSwThermalSlowdown",
             "sw_power_cap": "nvmlClocksEventReasonSwPowerCap",
             "hw_power_brake": "nvmlClocksEventReasonHwPowerBrakeSlowdown"}

    def __init__(self, index: int):
        self.index = index
        self.sm: list[float] = []
        self.reasons: set[str] = set()
        self.smax = None
        self.err = None
        self._stop = threading.Event()
        self.t = None

    def start(self):
        try:
            import pynvml as nv

            nv.nvmlInit()
            self.nv = nv
            self.h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.smax = float(nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM))
            self.masks = {k: getattr(nv, v, 0) for k, v in self.NAMES.items()}
        except Exception as e:  # noqa: BLE001
            self.err = f"nvml unavailable: {e}"
            return
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.sm.append(float(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, m in self.masks.items():
                    if m and (r & m):
                        self.reasons.add(k)
            except Exception as e:  # noqa: BLE001
                self.err = str(e)
                return
            time.sleep(0.002)

    def stop(self) -> dict:
        if self.t is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [self.err or "not sampled"], "samples": 0}
        self._stop.set()
        self.t.join(timeout=5)
        loaded = [x for x in self.sm if self.smax and x > 0.5 * self.smax] or self.sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": self.smax,
                "reasons": sorted(self.reasons), "samples": len(self.sm)}


def workload(cfg_name: str):
    import synth

    c = synth.CONFIGS[cfg_name]
    fields = c.get("fields", [None])
    return c, fields, c["rel"]


# ---------------------------------------------------------------- reference arm

METRIC = "end-to-end compress+decompress GB/s (input fp32), REL, incl. range kernel"
REF_SAMPLE = 1 << 20      # elements per field in each reference step


def run_reference(args, rank, world):
    """The CPU oracle, as it stands, on a bounded sample of the same workload:
    every step runs the same round-trip mix as our arm (every field x every
    REL bound) on the first REF_SAMPLE elements of each field."""
    if rank != 0:
        return
    import oracle
    import synth

    oracle.build()
    c, fields, rels = workload(args.config)
    samples = {}
    for f in fields:
        x = synth.field_for_config(args.config, device="cpu", field=f).numpy()
        samples[f] = x[: min(x.size, REF_SAMPLE)].copy()
    t_steps = []
    n_step = 0
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        n_step = 0
        for f in fields:
            for rel in rels:
                st, s = oracle.compress(samples[f], rel, oracle.REL)
                st2, y = oracle.decompress(s, samples[f].size)
                assert st == st2 == oracle.OK
                n_step += samples[f].size
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            t_steps.append(dt)
    tot = sum(t_steps)
    gbs = n_step * 4 * len(t_steps) / tot / 1e9
    sample = f"first {REF_SAMPLE} elements of each field ({', '.join(f for f in fields if f)}) x REL {rels}"
    line = {
        "impl": "reference", "metric": METRIC, "value": gbs,
        "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": tot / len(t_steps) * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": args.config, "fields": [f for f in fields if f] or None, "rel": rels,
                   "round_trips_per_step": len(fields) * len(rels), "sample": sample},
        "cpu_baseline": {"value": gbs, "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": sample + ", single-threaded C++ oracle, all round trips of a step"},
        "e2e": {"value": gbs, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# -------------------------------------------------------------------- our arm

def cpu_baseline(args, cfg_name, fields, rels):
    import oracle
    import synth

    oracle.build()
    x = synth.field_for_config(cfg_name, device="cpu", field=fields[0]).numpy()
    rel = rels[len(rels) // 2]
    n_done, t_tot, reps = 0, 0.0, 0
    while t_tot < args.cpu_seconds or reps == 0:
        t0 = time.perf_counter()
        st, s = oracle.compress(x, rel, oracle.REL)
        st2, y = oracle.decompress(s, x.size)
        t_tot += time.perf_counter() - t0
        n_done += x.size
        reps += 1
    return {"value": n_done * 4 / t_tot / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": f"{reps} round trip(s) of {cfg_name}/{fields[0]} ({x.size} elements) at REL {rel}, "
                      f"{t_tot:.1f} s single-threaded C++ oracle"}


def run_ours(args, rank, world, dev):
    import paper_conf_sc_huangd0lc23_b200 as cz
    import synth
    from paper_conf_sc_huangd0lc23_b200 import dist as czd

    lib = cz.lib()
    c, fields, rels = workload(args.config)
    stream = torch.cuda.current_stream(dev)
    sp = int(stream.cuda_stream)

    # ---- inputs resident in HBM (generated on the device, seeded per rank)
    xs = {}
    for f in fields:
        xs[f] = synth.field_for_config(args.config, device=dev, field=f)
        if world > 1 and rank > 0:
            xs[f] = xs[f].roll(rank * 4099)      # distinct data per rank, same statistics
    n_of = {f: xs[f].numel() for f in fields}
    nmax = max(n_of.values())
    ws = cz.Workspace(nmax, dev)
    cap = cz.max_compressed_bytes(nmax)
    out = torch.empty(cap, dtype=torch.uint8, device=dev)
    out_bytes = torch.zeros(1, dtype=torch.int64, device=dev)
    y = torch.empty(nmax, dtype=torch.float32, device=dev)
    mm_local = torch.empty(2, dtype=torch.float32, device=dev)
    mm_all = torch.empty(2 * world, dtype=torch.float32, device=dev)
    flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    sink = torch.empty(1, dtype=torch.int64, device=dev)

    def flush_l2():
        # write then read 512 MB (> 126 MB L2): the L2 ends up holding CLEAN lines
        # of an unrelated buffer -- a write-only flush would leave ~126 MB of
        # dirty lines whose write-back gets charged to the next timed kernel
        flush_buf.zero_()
        sink.copy_(flush_buf.view(torch.int64).sum())

    jobs = [(f, r) for f in fields for r in rels]
    group = torch.distributed.group.WORLD if world > 1 else None

    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in jobs]
    acc = {"range": 0.0, "compress": 0.0, "decompress": 0.0}
    sizes = {}

    def one_step(timed: bool):
        for j, (f, rel) in enumerate(jobs):
            x = xs[f]
            n = n_of[f]
            flush_l2()                                      # L2 flush, untimed
            e = ev[j]
            e[0].record(stream)
            cz.check(lib.cuszp_range(x.data_ptr(), n, mm_local.data_ptr(), ws.ptr(), ws.nbytes, sp), "range")
            if world > 1:
                czd.allgather_minmax(mm_local, mm_all, group)   # global REL range over NVLink
                mm, pairs = mm_all, world
            else:
                mm, pairs = mm_local, 1
            e[1].record(stream)
            cz.check(lib.cuszp_compress_minmax(x.data_ptr(), n, float(rel), mm.data_ptr(), pairs, out.data_ptr(),
                                               cap, out_bytes.data_ptr(), ws.ptr(), ws.nbytes, sp), "compress")
            if world > 1:
                czd.allgather_sizes(out_bytes, group)          # container header offsets
            e[2].record(stream)
            cz.check(lib.cuszp_decompress(out.data_ptr(), cap, y.data_ptr(), n, ws.ptr(), ws.nbytes, sp),
                     "decompress")
            e[3].record(stream)
            if timed:
                torch.cuda.synchronize(dev)
                acc["range"] += e[0].elapsed_time(e[1])
                acc["compress"] += e[1].elapsed_time(e[2])
                acc["decompress"] += e[2].elapsed_time(e[3])
                sizes[(f, rel)] = int(out_bytes.item())

    for _ in range(max(args.warmup, 3)):
        one_step(False)
    torch.cuda.synchronize(dev)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize(dev)
    clocks = ClockSampler(dev.index)
    clocks.start()
    t_wall0 = time.perf_counter()
    for _ in range(args.steps):
        one_step(True)
    torch.cuda.synchronize(dev)
    t_wall = time.perf_counter() - t_wall0
    clk = clocks.stop()
    if world > 1:
        torch.distributed.barrier()

    # verification of every round trip on the device with the fused quality
    # kernel (cuszp_quality; untimed): the bound of
    # DESIGN sec 5, PSNR per job, and the quality kernel's own HBM rate
    quality = {"psnr": {}, "max_abs_err_over_eb": {}}
    qev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    q_ms = []
    for f, rel in jobs:
        x = xs[f]
        n = n_of[f]
        cz.check(lib.cuszp_range(x.data_ptr(), n, mm_local.data_ptr(), ws.ptr(), ws.nbytes, sp), "range")
        cz.check(lib.cuszp_compress_minmax(x.data_ptr(), n, float(rel), mm_local.data_ptr(), 1, out.data_ptr(),
                                           cap, out_bytes.data_ptr(), ws.ptr(), ws.nbytes, sp), "compress")
        cz.check(lib.cuszp_decompress(out.data_ptr(), cap, y.data_ptr(), n, ws.ptr(), ws.nbytes, sp), "decompress")
        hdr = cz.read_header(out)
        assert hdr["status"] == 0 and cz.last_status(ws) == cz.OK
        flush_l2()
        qev[0].record(stream)
        qraw = cz.quality(x, y[:n], bound=float(hdr["eb_abs"]), sync=False)
        qev[1].record(stream)
        torch.cuda.synchronize(dev)
        q_ms.append(qev[0].elapsed_time(qev[1]))
        qv = qraw.cpu()
        ulp_max = float(np.spacing(np.float32(max(abs(qv[0].item()), abs(qv[1].item())))))
        assert qv[3].item() <= hdr["eb_abs"] + ulp_max, (f, rel, qv[3].item(), hdr["eb_abs"])
        quality["psnr"][f"{f}@{rel:g}"] = round(qv[7].item(), 3)
        quality["max_abs_err_over_eb"][f"{f}@{rel:g}"] = round(qv[3].item() / hdr["eb_abs"], 6)
    q_bytes = sum(8 * n_of[f] for f, _ in jobs)
    quality["kernel_gbs"] = q_bytes / (sum(q_ms) / 1e3) / 1e9

    # a large field (HACC-shaped, 1.12 GB, REL 1e-3; BASELINE configs[2]) where
    # launch ramp and drain are amortised: kernel times and roofline fractions
    # (context for the 100 MB headline fields; inputs >> L2, median of 3)
    large = None
    if not args.no_large and world == 1:
        xl = synth.field_for_config("c3_hacc", device=dev)
        nl = xl.numel()
        capl = cz.max_compressed_bytes(nl)
        wsl = cz.Workspace(nl, dev)
        outl = torch.empty(capl, dtype=torch.uint8, device=dev)
        yl = torch.empty(nl, dtype=torch.float32, device=dev)
        mml = torch.empty(2, dtype=torch.float32, device=dev)
        tl = {"range": [], "compress": [], "decompress": []}
        ev4 = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        for _ in range(4):
            ev4[0].record(stream)
            cz.check(lib.cuszp_range(xl.data_ptr(), nl, mml.data_ptr(), wsl.ptr(), wsl.nbytes, sp), "range")
            ev4[1].record(stream)
            cz.check(lib.cuszp_compress_minmax(xl.data_ptr(), nl, 1e-3, mml.data_ptr(), 1, outl.data_ptr(), capl,
                                               out_bytes.data_ptr(), wsl.ptr(), wsl.nbytes, sp), "compress")
            ev4[2].record(stream)
            cz.check(lib.cuszp_decompress(outl.data_ptr(), capl, yl.data_ptr(), nl, wsl.ptr(), wsl.nbytes, sp),
                     "decompress")
            ev4[3].record(stream)
            torch.cuda.synchronize(dev)
            for k, (e0, e1) in zip(tl, ((0, 1), (1, 2), (2, 3))):
                tl[k].append(ev4[e0].elapsed_time(ev4[e1]) / 1e3)
        assert cz.last_status(wsl) == cz.OK
        Sl = int(out_bytes.item())
        med = {k: float(np.median(v[1:])) for k, v in tl.items()}
        bl = {"range": 4 * nl, "compress": 4 * nl + Sl, "decompress": Sl + 4 * nl}
        large = {"workload": "c3_hacc (280,953,867 fp32, 1.12 GB) REL 1e-3", "cr": round(4 * nl / Sl, 3),
                 **{k: {"us": round(med[k] * 1e6, 1), "algorithmic_gbs": round(bl[k] / med[k] / 1e9, 1),
                        "frac_of_peak": round(bl[k] / med[k] / 1e9 / peak_hbm()[0], 4)} for k in med}}
        del xl, yl, outl, wsl
        torch.cuda.empty_cache()

    # block-length variants on the first field at the
    # middle bound: compress and decompress kernels, L2 flushed, median of 5
    f0, rel0 = fields[0], rels[len(rels) // 2]
    x0, n0 = xs[f0], n_of[f0]
    cz.check(lib.cuszp_range(x0.data_ptr(), n0, mm_local.data_ptr(), ws.ptr(), ws.nbytes, sp), "range")
    variants = {}
    for Lb, order in ((8, 1), (16, 1), (32, 1), (64, 1), (128, 1), (32, 2)):
        tc, td = [], []
        capL = cz.max_compressed_bytes(n0, Lb)
        outL = out if capL <= cap else torch.empty(capL, dtype=torch.uint8, device=dev)
        for _ in range(6):
            flush_l2()
            qev[0].record(stream)
            if order == 1:
                cz.check(lib.cuszp_compress_minmax_L(x0.data_ptr(), n0, float(rel0), mm_local.data_ptr(), 1, Lb,
                                                     outL.data_ptr(), capL, out_bytes.data_ptr(), ws.ptr(), ws.nbytes,
                                                     sp), "compress_L")
            else:   # 2-layer Lorenzo: REL through the range kernel too
                cz.check(lib.cuszp_compress_ex(x0.data_ptr(), n0, float(rel0), cz.REL, Lb, order, outL.data_ptr(),
                                               capL, out_bytes.data_ptr(), ws.ptr(), ws.nbytes, sp), "compress_ex")
            qev[1].record(stream)
            torch.cuda.synchronize(dev)
            tc.append(qev[0].elapsed_time(qev[1]))
            flush_l2()
            qev[0].record(stream)
            cz.check(lib.cuszp_decompress_ex(outL.data_ptr(), capL, y.data_ptr(), n0, Lb, order, ws.ptr(),
                                             ws.nbytes, sp), "decompress_ex")
            qev[1].record(stream)
            torch.cuda.synchronize(dev)
            td.append(qev[0].elapsed_time(qev[1]))
        assert cz.last_status(ws) == cz.OK
        SL = int(out_bytes.item())
        tcm, tdm = float(np.median(tc[1:])) / 1e3, float(np.median(td[1:])) / 1e3
        variants[str(Lb) if order == 1 else f"{Lb}_lorenzo2"] = {"cr": round(4 * n0 / SL, 3),
                             "compress_kernel_gbs": round(4 * n0 / tcm / 1e9, 1),
                             "decompress_kernel_gbs": round(4 * n0 / tdm / 1e9, 1),
                             "compress_frac_of_peak": round((4 * n0 + SL) / tcm / 1e9 / peak_hbm()[0], 4),
                             "decompress_frac_of_peak": round((4 * n0 + SL) / tdm / 1e9 / peak_hbm()[0], 4)}

    t_dev = torch.tensor([acc["range"], acc["compress"], acc["decompress"]], dtype=torch.float64, device=dev)
    if world > 1:
        torch.distributed.all_reduce(t_dev, op=torch.distributed.ReduceOp.MAX)
    t_range, t_comp, t_decomp = (float(v) / 1e3 for v in t_dev.tolist())   # seconds over K steps
    K = args.steps
    in_bytes_step = sum(4 * n_of[f] for f, _ in jobs)
    total_bytes = in_bytes_step * K * world
    t_step_total = t_range + t_comp + t_decomp
    S = {k: v for k, v in sizes.items()}
    cr = {f"{f}@{r:g}": round(4 * n_of[f] / S[(f, r)], 3) for f, r in jobs}

    peak, peak_src = peak_hbm()
    per_launch = {
        "range": sum(4 * n_of[f] for f, _ in jobs) / (t_range / K),
        "compress": sum(4 * n_of[f] + S[(f, r)] for f, r in jobs) / (t_comp / K),
        "decompress": sum(S[(f, r)] + 4 * n_of[f] for f, r in jobs) / (t_decomp / K),
    }
    times = {"range": t_range, "compress": t_comp, "decompress": t_decomp}
    dom = max(times, key=times.get)
    achieved = per_launch[dom] / 1e9
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as fh:
            traffic = json.load(fh).get("dram_bytes_per_launch", {}).get(dom)
    except Exception:
        pass

    line = {
        "metric": METRIC,
        "value": total_bytes / t_step_total / 1e9 / K * K,
        "unit": "GB/s", "n_gpus": world, "steps": K, "warmup": max(args.warmup, 3),
        "ms_per_step": t_step_total / K * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": args.config, "fields": [f for f in fields if f] or None, "rel": rels,
                   "n_per_field": n_of[fields[0]], "round_trips_per_step": len(jobs),
                   "parallelism": f"dp{world}" if world > 1 else "single",
                   "l2": "flushed (512 MB write + read, untimed) before every round trip"},
        "compress_gbs": in_bytes_step * K * world / (t_range + t_comp) / 1e9,
        "compress_kernel_only_gbs": in_bytes_step * K * world / t_comp / 1e9,
        "decompress_gbs": in_bytes_step * K * world / t_decomp / 1e9,
        "cr": cr,
        "kernels": {k: {"ms_per_step": times[k] / K * 1e3, "algorithmic_gbs": per_launch[k] / 1e9,
                        "frac_of_peak": per_launch[k] / 1e9 / peak} for k in times},
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src},
        "gpu_launches": 3 * len(jobs) * K,
        "block_len_variants": {"workload": f"{f0}@{rel0:g}", "unit": "GB/s of fp32 input", **variants},
        "large_field": large,
        "quality": dict(quality, frac_of_peak=quality["kernel_gbs"] / peak,
                        kernel="cuszp_quality (fused compareData statistics, untimed verification pass)"),
        "clocks": clk,
        "wall_s_timed_region": t_wall,
        "paper_context": PAPER_A100,
    }

    # ---- e2e through the asynchronous host-buffer C-ABI calls (pinned memory):
    # every job H2D-copies its field, compresses, moves the stream into host
    # memory (exactly S bytes, SM copy kernel reading the device-side length),
    # brings it back, decompresses and D2H-copies the reconstruction; jobs
    # rotate over three streams so one job's device->host traffic overlaps
    # the next jobs' host->device traffic on the link.
    if not args.no_e2e:
        h_in = {f: xs[f].cpu().pin_memory() for f in fields}
        lanes = []
        n_lanes = int(os.environ.get("CUSZP_E2E_LANES", "3"))
        for _ in range(n_lanes):
            lanes.append(dict(stream=torch.cuda.Stream(dev),
                              h_out=torch.zeros(cap, dtype=torch.uint8).pin_memory(),
                              h_len=torch.zeros(1, dtype=torch.int64).pin_memory(),
                              h_y=torch.empty(nmax, dtype=torch.float32).pin_memory(),
                              d_in=torch.empty(nmax, dtype=torch.float32, device=dev),
                              d_out=torch.empty(cap, dtype=torch.uint8, device=dev),
                              d_y=torch.empty(nmax, dtype=torch.float32, device=dev),
                              ws=cz.Workspace(nmax, dev)))
        h2d = d2h = 0
        lens = {}
        for i in range(1 + args.steps):
            if i == 1:
                torch.cuda.synchronize(dev)
                if world > 1:
                    torch.distributed.barrier()
                t0 = time.perf_counter()
            for j, (f, rel) in enumerate(jobs):
                ln = lanes[j % n_lanes]
                n = n_of[f]
                cz.compress_host_async(h_in[f], rel, "rel", ln["h_out"], ln["h_len"], ln["d_in"], ln["d_out"],
                                       ln["ws"], stream=ln["stream"])
                cz.decompress_host_async(ln["h_out"], ln["h_y"][:n], ln["d_out"], ln["d_y"], ln["ws"],
                                         stream=ln["stream"])
                if i == 0:      # warm-up pass: record the stream lengths (bytes counted per step)
                    ln["stream"].synchronize()
                    lens[(f, rel)] = int(ln["h_len"].item())
        torch.cuda.synchronize(dev)
        t_e2e = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        if world > 1:
            torch.distributed.all_reduce(t_e2e, op=torch.distributed.ReduceOp.MAX)
        for f, rel in jobs:
            n = n_of[f]
            h2d += 4 * n + lens[(f, rel)]              # field in, stream back in
            d2h += lens[(f, rel)] + 8 + 4 * n          # stream + its length out, reconstruction out
        # the last job's reconstruction in host memory satisfies the bound
        f_l, rel_l = jobs[-1]
        ln = lanes[(len(jobs) - 1) % n_lanes]
        eb_l = float(np.frombuffer(ln["h_out"][16:20].numpy().tobytes(), np.float32)[0])
        err = (ln["h_y"][: n_of[f_l]].double() - h_in[f_l].double()).abs().max().item()
        assert err <= eb_l + float(np.spacing(np.float32(h_in[f_l].abs().max().item()))), (err, eb_l)
        # the host link's own ceiling for this traffic: both directions at once (copy engines)
        pa = torch.empty(1 << 28, dtype=torch.uint8).pin_memory()
        pb = torch.empty(1 << 28, dtype=torch.uint8).pin_memory()
        da = torch.empty(1 << 28, dtype=torch.uint8, device=dev)
        db = torch.empty(1 << 28, dtype=torch.uint8, device=dev)
        def both_ways():
            with torch.cuda.stream(lanes[0]["stream"]):
                da.copy_(pa, non_blocking=True)
            with torch.cuda.stream(lanes[1]["stream"]):
                pb.copy_(db, non_blocking=True)
        both_ways()                                     # first touch of the pinned pages, untimed
        torch.cuda.synchronize(dev)
        tl0 = time.perf_counter()
        for _ in range(4):
            both_ways()
        torch.cuda.synchronize(dev)
        link_gbs = 4 * (1 << 28) / (time.perf_counter() - tl0) / 1e9     # per direction
        e2e_bound = in_bytes_step / (max(h2d, d2h) / (link_gbs * 1e9)) / 1e9 * world
        line["e2e"] = {"value": in_bytes_step * K * world / float(t_e2e.item()) / 1e9, "unit": "GB/s",
                       "link_gbs_per_direction": round(link_gbs, 1), "link_bound_gbs": round(e2e_bound, 1),
                       "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                       "path": "cuszp_compress_host_async + cuszp_decompress_host_async (pinned host buffers, "
                               f"{n_lanes} streams, wall clock)"}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(args, args.config, fields, rels)
    return line


def main():
    args = parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    # CUSZP_BENCH_SHARE_GPU=1 (diagnostics only): every rank on the same GPU
    # over gloo, to exercise the N > 1 code path on a one-GPU box
    share = os.environ.get("CUSZP_BENCH_SHARE_GPU") == "1"
    dev = torch.device("cuda", local % torch.cuda.device_count() if share else local)
    torch.cuda.set_device(dev)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if share:
            torch.distributed.init_process_group("gloo")
        else:
            torch.distributed.init_process_group("nccl", device_id=dev)
    line = run_ours(args, rank, world, dev)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
