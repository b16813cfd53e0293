#!/usr/bin/env python
"""bench.py -- throughput of the cuSZp hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N --steps K --warmup W] [--impl ours|reference]
                    [--config c3_hacc|c5_rtm|c1_smooth1d|c2_hurricane|c4_nyx]

A STEP is one pass of the whole hot path over one
batch of synthetic input: for every field of the config and every REL bound
it names, value range (a1) -> fused compression (a2..a8) -> fused
decompression (a9..a12), all through the C ABI.

Workload (config.workload):
  N = 1  the largest single-GPU configuration of BASELINE.json, configs[2]:
         the HACC-shaped 1D field, 280,953,867 fp32 (1.124 GB), REL 1e-3
         (default --config c3_hacc);
  N > 1  configs[4]: ONE RTM-shaped 6.82 GB snapshot set (36 x 449x449x235
         fp32) SHARDED across the N ranks in block-aligned slabs (the
         north_star split): rank p compresses its slab against the
         GLOBAL range (NCCL all-gather of 8 B per rank) and the compressed
         byte counts are all-gathered into the container header (8 B per
         rank) -- both exchanges inside the timed region (default
         --config c5_rtm; "scaling": "strong", total work fixed).
The other configs are reported as secondary keys at N = 1 (c1 as a CUDA-graph
replay, c2's 9 round trips, c4, and c5 on one GPU).

Timing: the L2 (126 MB) is flushed (a 512 MB write + read, untimed) before
every round trip; each kernel is bracketed by CUDA events on the launching
stream; a step's time is the sum of its kernels' device time (max over
ranks).  W warm-up steps, then K timed steps between barrier + synchronize.

--impl reference runs the CPU oracle (oracle/, single thread) on a bounded
sample of the same workload -- the tier's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import statistics
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
METRIC = "end-to-end compress+decompress GB/s (input fp32), REL, incl. range kernel"
REF_SAMPLE = 1 << 24      # elements per field in each reference step (16 windows of 2^20)


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default=None, help="default: c3_hacc at N = 1, c5_rtm (sharded) at N > 1")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-secondary", action="store_true", help="skip the c1/c2/c4/c5 secondary keys")
    p.add_argument("--no-variants", action="store_true", help="skip the block-length / predictor variants")
    p.add_argument("--no-datasets", action="store_true", help="skip the six-dataset table")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=12.0)
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


def host_info() -> dict:
    model = platform.processor() or ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


class ClockSampler:
    """SM clock + clock-event (throttle) reasons polled through NVML every
    ~2 ms from a thread while the timed region runs."""
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


def resolve_config(args, world: int) -> str:
    return args.config or ("c3_hacc" if world == 1 else "c5_rtm")


def config_jobs(cfg_name: str):
    import synth

    c = synth.CONFIGS[cfg_name]
    fields = c.get("fields", [None])
    return fields, c["rel"]


def make_field(cfg_name: str, field, device):
    import synth

    return synth.field_for_config(cfg_name, device=device, field=field)


def slab(n: int, rank: int, world: int):
    from paper_conf_sc_huangd0lc23_b200 import dist as czd

    return czd.slab_bounds(n, rank, world)


# ---------------------------------------------------------------- reference arm

def run_reference(args, rank, world):
    """The CPU oracle, as it stands, on a bounded sample of the same workload:
    every step runs the round trips of our arm's step (every field x every
    REL bound) on REF_SAMPLE elements of each field, taken as 16 evenly spaced
    2^20-element windows (block aligned) so sparse and dense parts are both
    represented (RTM's first snapshots are nearly all zero)."""
    if rank != 0:
        return
    import oracle

    oracle.build()
    cfg = resolve_config(args, world)
    fields, rels = config_jobs(cfg)
    gen_dev = "cuda" if torch.cuda.is_available() else "cpu"
    samples = {}
    for f in fields:
        x = make_field(cfg, f, gen_dev)
        n = x.numel()
        if n <= REF_SAMPLE:
            samples[f] = x.cpu().numpy()
        else:
            w = REF_SAMPLE // 16
            starts = [((k * (n - w)) // 15) // 32 * 32 for k in range(16)]
            samples[f] = torch.cat([x[s:s + w] for s in starts]).cpu().numpy()
        del x
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
    sample = (f"{min(REF_SAMPLE, samples[fields[0]].size)} elements of each field "
              f"({', '.join(f for f in fields if f) or cfg}; 16 evenly spaced windows) x REL {rels}")
    line = {
        "impl": "reference", "metric": METRIC, "value": gbs,
        "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": tot / len(t_steps) * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfg, "fields": [f for f in fields if f] or None, "rel": rels,
                   "round_trips_per_step": len(fields) * len(rels), "sample": sample},
        "cpu_baseline": {"value": gbs, "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": sample + ", single-threaded C++ oracle, all round trips of a step",
                         "host": host_info()},
        "e2e": {"value": gbs, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# -------------------------------------------------------------------- our arm

class Runner:
    """Device buffers + timing of round trips through the C ABI."""

    def __init__(self, dev, nmax: int, world: int = 1, group=None):
        import paper_conf_sc_huangd0lc23_b200 as cz

        self.cz = cz
        self.lib = cz.lib()
        self.dev = dev
        self.world = world
        self.group = group
        self.stream = torch.cuda.current_stream(dev)
        self.sp = int(self.stream.cuda_stream)
        self.ws = cz.Workspace(max(nmax, 1), dev)
        self.cap = cz.max_compressed_bytes(nmax)
        self.out = torch.empty(self.cap, dtype=torch.uint8, device=dev)
        self.out_bytes = torch.zeros(1, dtype=torch.int64, device=dev)
        self.y = torch.empty(max(nmax, 1), dtype=torch.float32, device=dev)
        self.mm_local = torch.empty(2, dtype=torch.float32, device=dev)
        self.mm_all = torch.empty(2 * world, dtype=torch.float32, device=dev)
        self.sizes_all = torch.empty(world, dtype=torch.int64, device=dev)
        self.flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
        self.sink = torch.empty(1, dtype=torch.int64, device=dev)

    def flush_l2(self):
        # write then read 512 MB (> 126 MB L2): the L2 ends up holding CLEAN lines
        # of an unrelated buffer -- a write-only flush would leave ~126 MB of
        # dirty lines whose write-back gets charged to the next timed kernel
        self.flush_buf.zero_()
        self.sink.copy_(self.flush_buf.view(torch.int64).sum())

    def round_trip(self, x, n, rel, ev=None):
        """range -> (all-gather of (min,max)) -> compress -> (all-gather of
        sizes) -> decompress, events between the stages."""
        cz, lib, sp = self.cz, self.lib, self.sp
        from paper_conf_sc_huangd0lc23_b200 import dist as czd

        if ev is not None:
            ev[0].record(self.stream)
        cz.check(lib.cuszp_range(x.data_ptr(), n, self.mm_local.data_ptr(), self.ws.ptr(), self.ws.nbytes, sp),
                 "range")
        if self.world > 1:
            czd.allgather_minmax(self.mm_local, self.mm_all, self.group)   # global REL range (NVLink)
            mm, pairs = self.mm_all, self.world
        else:
            mm, pairs = self.mm_local, 1
        if ev is not None:
            ev[1].record(self.stream)
        cz.check(lib.cuszp_compress_minmax(x.data_ptr(), n, float(rel), mm.data_ptr(), pairs, self.out.data_ptr(),
                                           self.cap, self.out_bytes.data_ptr(), self.ws.ptr(), self.ws.nbytes, sp),
                 "compress")
        if self.world > 1:
            czd.allgather_sizes(self.out_bytes, self.group, self.sizes_all)   # container header offsets
        if ev is not None:
            ev[2].record(self.stream)
        cz.check(lib.cuszp_decompress(self.out.data_ptr(), self.cap, self.y.data_ptr(), n, self.ws.ptr(),
                                      self.ws.nbytes, sp), "decompress")
        if ev is not None:
            ev[3].record(self.stream)

    def measure(self, jobs, steps: int, warmup: int, clocks: ClockSampler | None = None):
        """jobs = [(label, x, n, rel)]; per-kernel device seconds summed over
        the timed steps (max over ranks), compressed sizes per job."""
        ev = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in jobs]
        acc = {"range": 0.0, "compress": 0.0, "decompress": 0.0}
        sizes = {}
        for _ in range(max(warmup, 3)):
            for lab, x, n, rel in jobs:
                self.flush_l2()
                self.round_trip(x, n, rel)
        torch.cuda.synchronize(self.dev)
        if self.world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize(self.dev)
        if clocks is not None:
            clocks.start()
        t0 = time.perf_counter()
        for _ in range(steps):
            for j, (lab, x, n, rel) in enumerate(jobs):
                self.flush_l2()                                   # L2 flush, untimed
                self.round_trip(x, n, rel, ev[j])
                torch.cuda.synchronize(self.dev)
                e = ev[j]
                acc["range"] += e[0].elapsed_time(e[1]) / 1e3
                acc["compress"] += e[1].elapsed_time(e[2]) / 1e3
                acc["decompress"] += e[2].elapsed_time(e[3]) / 1e3
                sizes[lab] = int(self.out_bytes.item())
                assert self.cz.read_header(self.out)["status"] == 0, lab
        torch.cuda.synchronize(self.dev)
        wall = time.perf_counter() - t0
        clk = clocks.stop() if clocks is not None else None
        if self.world > 1:
            torch.distributed.barrier()
        t = torch.tensor([acc["range"], acc["compress"], acc["decompress"]], dtype=torch.float64, device=self.dev)
        if self.world > 1:
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        acc = dict(zip(("range", "compress", "decompress"), (float(v) for v in t.tolist())))
        return acc, sizes, wall, clk


def summarise(jobs, acc, sizes, steps, world, peak, n_total=None):
    """Throughputs of a measured job list: GB/s of fp32 input (whole job),
    per-kernel algorithmic HBM bytes / time and the fraction of the peak."""
    in_bytes = sum(4 * n for _, _, n, _ in jobs)                  # this rank's input per step
    # whole-job input: every rank's slab of every job (n_total = elements per step, all ranks)
    in_total = (4 * n_total if n_total is not None else in_bytes * world) * steps
    t = acc["range"] + acc["compress"] + acc["decompress"]
    S = {lab: sizes[lab] for lab, *_ in jobs}
    alg = {"range": sum(4 * n for _, _, n, _ in jobs),
           "compress": sum(4 * n + S[lab] for lab, _, n, _ in jobs),
           "decompress": sum(S[lab] + 4 * n for lab, _, n, _ in jobs)}
    kernels = {k: {"us_per_step": acc[k] / steps * 1e6,
                   "algorithmic_gbs": alg[k] * steps / acc[k] / 1e9,
                   "frac_of_peak": alg[k] * steps / acc[k] / 1e9 / peak} for k in acc}
    return {
        "round_trip_gbs": in_total / t / 1e9,
        "compress_gbs": in_total / (acc["range"] + acc["compress"]) / 1e9,
        "compress_kernel_only_gbs": in_total / acc["compress"] / 1e9,
        "decompress_gbs": in_total / acc["decompress"] / 1e9,
        "rel_compress_frac_of_peak": (alg["range"] + alg["compress"]) * steps / (acc["range"] + acc["compress"])
        / 1e9 / peak,
        "cr": {lab: round(4 * n / S[lab], 3) for lab, _, n, _ in jobs},
        "kernels": kernels,
        "ms_per_step": t / steps * 1e3,
        "alg_bytes_per_step": alg,
    }


def cpu_baseline(x_np: np.ndarray, rel: float, seconds: float, label: str) -> dict:
    """The oracle as it stands on the same field: single-threaded round trips
    (the baseline proper, cores = 1), plus the same oracle run slab-parallel
    on every host core (block-aligned slabs against the global range; ctypes
    releases the GIL) as context."""
    import concurrent.futures as cf

    import oracle

    oracle.build()
    n = x_np.size
    n_done, t_tot, reps = 0, 0.0, 0
    while t_tot < seconds or reps == 0:
        t0 = time.perf_counter()
        st, s = oracle.compress(x_np, rel, oracle.REL)
        st2, y = oracle.decompress(s, n)
        t_tot += time.perf_counter() - t0
        assert st == st2 == oracle.OK
        n_done += n
        reps += 1
        del s, y
    hi = host_info()
    P = max(1, int(hi["nproc"] or 1))
    lo_, hi_ = oracle.value_range(x_np)
    mm = np.array([lo_, hi_], np.float32)

    def part(p):
        s0, s1 = slab(n, p, P)
        st, s = oracle.compress_minmax(x_np[s0:s1], rel, mm)
        st2, y = oracle.decompress(s, s1 - s0)
        return st == st2 == oracle.OK

    t0 = time.perf_counter()
    oracle.value_range(x_np)
    with cf.ThreadPoolExecutor(P) as ex:
        assert all(ex.map(part, range(P)))
    t_all = time.perf_counter() - t0
    return {"value": n_done * 4 / t_tot / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": f"{reps} full round trip(s) of {label} ({n} elements) at REL {rel}: oracle value range + "
                      f"compress + decompress, {t_tot:.1f} s single-threaded C++ oracle (-O2)",
            "host": hi,
            "all_cores": {"value": 4 * n / t_all / 1e9, "unit": "GB/s", "cores": P,
                          "how": f"the same oracle on {P} block-aligned slabs in {P} threads (global range)"}}


def e2e_measure(cz, dev, jobs_host, steps: int, world: int, cap: int, nmax: int) -> dict:
    """End to end through the asynchronous host-buffer C-ABI calls (pinned
    memory): every job H2D-copies its field, compresses, moves the stream into
    host memory (exactly S bytes, SM copy kernel reading the device-side
    length), brings it back, decompresses and D2H-copies the reconstruction;
    consecutive jobs rotate over streams so one job's device->host traffic
    overlaps the next one's host->device traffic.  Wall clock, max over ranks."""
    # Compressions run on "C" streams (host->device heavy: the field in, the
    # stream out) and decompressions on "D" streams (the stream in, the field
    # out), each job's decompression event-ordered after its compression, so
    # the two directions of the link carry balanced traffic at all times.
    n_sets = int(os.environ.get("CUSZP_E2E_LANES", "2"))
    # host stream buffers per set: with 2, a compression only waits for the
    # decompression that read the same buffer two rounds ago
    n_hbuf = int(os.environ.get("CUSZP_E2E_HBUF", "1"))
    sets = []
    for _ in range(n_sets):
        sets.append(dict(cs=torch.cuda.Stream(dev), ds=torch.cuda.Stream(dev),
                         h_outs=[torch.zeros(cap, dtype=torch.uint8).pin_memory() for _ in range(n_hbuf)],
                         dec_dones=[torch.cuda.Event() for _ in range(n_hbuf)], hb_used=[False] * n_hbuf, use=0,
                         h_len=torch.zeros(1, dtype=torch.int64).pin_memory(),
                         h_y=torch.empty(nmax, dtype=torch.float32).pin_memory(),
                         d_in=torch.empty(nmax, dtype=torch.float32, device=dev),
                         d_out=torch.empty(cap, dtype=torch.uint8, device=dev),
                         d_sin=torch.empty(cap, dtype=torch.uint8, device=dev),
                         d_y=torch.empty(nmax, dtype=torch.float32, device=dev),
                         wsc=cz.Workspace(nmax, dev), wsd=cz.Workspace(nmax, dev),
                         comp_done=torch.cuda.Event(), dec_done=torch.cuda.Event(), used=False))
    lens = {}
    k = 0
    for i in range(1 + steps):
        if i == 1:
            torch.cuda.synchronize(dev)
            if world > 1:
                torch.distributed.barrier()
            t0 = time.perf_counter()
        for lab, h_in, rel in jobs_host:
            st = sets[k % n_sets]
            k += 1
            n = h_in.numel()
            b = st["use"] % n_hbuf
            st["use"] += 1
            st["h_out"] = st["h_outs"][b]
            if st["hb_used"][b]:
                st["cs"].wait_event(st["dec_dones"][b])      # h_out is free once the decompression that read it is done
            cz.compress_host_async(h_in, rel, "rel", st["h_out"], st["h_len"], st["d_in"][:n], st["d_out"],
                                   st["wsc"], stream=st["cs"])
            st["comp_done"].record(st["cs"])
            st["ds"].wait_event(st["comp_done"])
            cz.decompress_host_async(st["h_out"], st["h_y"][:n], st["d_sin"], st["d_y"][:n], st["wsd"],
                                     stream=st["ds"])
            st["dec_dones"][b].record(st["ds"])
            st["hb_used"][b] = True
            if i == 0:      # warm-up pass: record the stream lengths (bytes counted per step)
                st["ds"].synchronize()
                lens[lab] = int(st["h_len"].item())
    n_lanes = 2 * n_sets
    torch.cuda.synchronize(dev)
    t_e2e = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
    if world > 1:
        torch.distributed.all_reduce(t_e2e, op=torch.distributed.ReduceOp.MAX)
    h2d = d2h = 0
    for lab, h_in, rel in jobs_host:
        n = h_in.numel()
        h2d += 4 * n + lens[lab]              # field in, stream back in
        d2h += lens[lab] + 8 + 4 * n          # stream + its length out, reconstruction out
    # the last job's reconstruction in host memory satisfies the bound
    lab, h_in, rel = jobs_host[-1]
    ln = sets[(k - 1) % n_sets]
    n = h_in.numel()
    eb_l = float(np.frombuffer(ln["h_out"][16:20].numpy().tobytes(), np.float32)[0])
    err = (ln["h_y"][:n].double() - h_in.double()).abs().max().item()
    assert err <= eb_l + float(np.spacing(np.float32(h_in.abs().max().item()))), (err, eb_l)
    del sets
    # the host link's own ceiling for this traffic: both directions at once (copy engines)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    pa = torch.empty(1 << 28, dtype=torch.uint8).pin_memory()
    pb = torch.empty(1 << 28, dtype=torch.uint8).pin_memory()
    da = torch.empty(1 << 28, dtype=torch.uint8, device=dev)
    db = torch.empty(1 << 28, dtype=torch.uint8, device=dev)

    def both_ways():
        with torch.cuda.stream(s1):
            da.copy_(pa, non_blocking=True)
        with torch.cuda.stream(s2):
            pb.copy_(db, non_blocking=True)

    both_ways()                                     # first touch of the pinned pages, untimed
    torch.cuda.synchronize(dev)
    tl0 = time.perf_counter()
    for _ in range(4):
        both_ways()
    torch.cuda.synchronize(dev)
    link_gbs = 4 * (1 << 28) / (time.perf_counter() - tl0) / 1e9     # per direction
    in_step = sum(4 * h.numel() for _, h, _ in jobs_host)
    bound = in_step / (max(h2d, d2h) / (link_gbs * 1e9)) / 1e9 * world
    return {"value": in_step * steps * world / float(t_e2e.item()) / 1e9, "unit": "GB/s",
            "link_gbs_per_direction": round(link_gbs, 1), "link_bound_gbs": round(bound, 1),
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "path": "cuszp_compress_host_async + cuszp_decompress_host_async (pinned host buffers; "
                    f"compressions and decompressions on {n_lanes} streams, event-ordered; wall clock)"}


def graph_replay_c1(r: Runner, steps: int, peak: float) -> dict:
    """c1 (2^20 elements, launch-bound) as a CUDA-graph replay of range +
    compress + decompress, L2 flushed before every replay."""
    x = make_field("c1_smooth1d", None, r.dev)
    n = x.numel()
    rel = config_jobs("c1_smooth1d")[1][0]
    s = torch.cuda.Stream(r.dev)
    s.wait_stream(torch.cuda.current_stream(r.dev))
    saved = (r.stream, r.sp)
    r.stream, r.sp = s, int(s.cuda_stream)
    with torch.cuda.stream(s):
        r.round_trip(x, n, rel)                          # library init outside capture
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        r.round_trip(x, n, rel)
    r.stream, r.sp = saved
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(3 + steps):
        r.flush_l2()
        torch.cuda.synchronize(r.dev)
        with torch.cuda.stream(s):
            e0.record(s)
            g.replay()
            e1.record(s)
        torch.cuda.synchronize(r.dev)
        if i >= 3:
            ts.append(e0.elapsed_time(e1) / 1e3)
    assert r.cz.read_header(r.out)["status"] == 0
    S = int(r.out_bytes.item())
    t = float(np.median(ts))
    # eager, same flush protocol, for comparison
    jobs = [("c1", x, n, rel)]
    acc, sizes, _, _ = r.measure(jobs, steps, 3)
    te = (acc["range"] + acc["compress"] + acc["decompress"]) / steps
    return {"workload": f"c1_smooth1d (2^20 fp32) REL {rel:g}", "cr": round(4 * n / S, 3),
            "graph_round_trip_us": round(t * 1e6, 2), "graph_round_trip_gbs": round(4 * n / t / 1e9, 1),
            "eager_round_trip_us": round(te * 1e6, 2), "eager_round_trip_gbs": round(4 * n / te / 1e9, 1),
            "note": "inputs fit in L2 (4 MB); flushed before every replay"}


def secondary(r: Runner, cfg: str, steps: int, peak: float) -> dict:
    fields, rels = config_jobs(cfg)
    xs = {f: make_field(cfg, f, r.dev) for f in fields}
    jobs = [(f"{f}@{rel:g}" if f else f"{rel:g}", xs[f], xs[f].numel(), rel) for f in fields for rel in rels]
    acc, sizes, _, _ = r.measure(jobs, steps, 3)
    d = summarise(jobs, acc, sizes, steps, 1, peak)
    jobs_n = jobs[0][2]
    del xs, jobs
    torch.cuda.empty_cache()
    return {"workload": cfg, "n_per_field": jobs_n, **{k: d[k] for k in (
        "round_trip_gbs", "compress_gbs", "decompress_gbs", "rel_compress_frac_of_peak", "cr", "kernels")}}


def variants(r: Runner, peak: float, steps: int) -> dict:
    """Block lengths L and the 2-layer predictor (rank 4)
    on Hurricane U at REL 1e-3, compress and decompress kernels only, eb from
    a given range (like for like: no range kernel in any of them), L2 flushed."""
    cz, lib, sp = r.cz, r.lib, r.sp
    x0 = make_field("c2_hurricane", "U", r.dev)
    n0 = x0.numel()
    rel0 = 1e-3
    cz.check(lib.cuszp_range(x0.data_ptr(), n0, r.mm_local.data_ptr(), r.ws.ptr(), r.ws.nbytes, sp), "range")
    mm = r.mm_local.cpu().numpy()
    eb_abs = float(np.float32(np.float32(rel0) * np.float32(mm[1] - mm[0])))
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    out = {"workload": f"c2_hurricane/U@{rel0:g}", "unit": "GB/s of fp32 input"}
    for Lb, order in ((8, 1), (16, 1), (32, 1), (64, 1), (128, 1), (32, 2)):
        tc, td = [], []
        capL = cz.max_compressed_bytes(n0, Lb)
        outL = r.out if capL <= r.cap else torch.empty(capL, dtype=torch.uint8, device=r.dev)
        for _ in range(steps + 1):
            r.flush_l2()
            ev[0].record(r.stream)
            if order == 1:
                cz.check(lib.cuszp_compress_minmax_L(x0.data_ptr(), n0, float(rel0), r.mm_local.data_ptr(), 1, Lb,
                                                     outL.data_ptr(), capL, r.out_bytes.data_ptr(), r.ws.ptr(),
                                                     r.ws.nbytes, sp), "compress_L")
            else:   # the same bound as ABS (the 2-layer path has no given-range entry point)
                cz.check(lib.cuszp_compress_ex(x0.data_ptr(), n0, eb_abs, cz.ABS, Lb, order, outL.data_ptr(),
                                               capL, r.out_bytes.data_ptr(), r.ws.ptr(), r.ws.nbytes, sp),
                         "compress_ex")
            ev[1].record(r.stream)
            torch.cuda.synchronize(r.dev)
            tc.append(ev[0].elapsed_time(ev[1]))
            r.flush_l2()
            ev[0].record(r.stream)
            cz.check(lib.cuszp_decompress_ex(outL.data_ptr(), capL, r.y.data_ptr(), n0, Lb, order, r.ws.ptr(),
                                             r.ws.nbytes, sp), "decompress_ex")
            ev[1].record(r.stream)
            torch.cuda.synchronize(r.dev)
            td.append(ev[0].elapsed_time(ev[1]))
        assert cz.last_status(r.ws) == cz.OK
        SL = int(r.out_bytes.item())
        tcm, tdm = float(np.median(tc[1:])) / 1e3, float(np.median(td[1:])) / 1e3
        out[str(Lb) if order == 1 else f"{Lb}_lorenzo2"] = {
            "cr": round(4 * n0 / SL, 3),
            "compress_kernel_gbs": round(4 * n0 / tcm / 1e9, 1),
            "decompress_kernel_gbs": round(4 * n0 / tdm / 1e9, 1),
            "compress_frac_of_peak": round((4 * n0 + SL) / tcm / 1e9 / peak, 4),
            "decompress_frac_of_peak": round((4 * n0 + SL) / tdm / 1e9 / peak, 4)}
        if outL is not r.out:
            del outL
    # multi-dimensional Lorenzo on the same field as
    # a (100, 500, 500) volume: 2D (1x4x8 blocks) and 3D (2x4x4 blocks)
    shape = (100, 500, 500)
    for dims in (2, 3):
        capm = int(lib.cuszp_max_compressed_bytes_md(*shape, dims))
        wsm = cz.WorkspaceMD(shape, dims, r.dev)
        outm = r.out if capm <= r.cap else torch.empty(capm, dtype=torch.uint8, device=r.dev)
        tc, td = [], []
        for _ in range(steps + 1):
            r.flush_l2()
            ev[0].record(r.stream)
            cz.check(lib.cuszp_compress_md(x0.data_ptr(), *shape, dims, eb_abs, cz.ABS, outm.data_ptr(), capm,
                                           r.out_bytes.data_ptr(), wsm.ptr(), wsm.nbytes, sp), "compress_md")
            ev[1].record(r.stream)
            torch.cuda.synchronize(r.dev)
            tc.append(ev[0].elapsed_time(ev[1]))
            r.flush_l2()
            ev[0].record(r.stream)
            cz.check(lib.cuszp_decompress_md(outm.data_ptr(), capm, r.y.data_ptr(), *shape, dims, wsm.ptr(),
                                             wsm.nbytes, sp), "decompress_md")
            ev[1].record(r.stream)
            torch.cuda.synchronize(r.dev)
            td.append(ev[0].elapsed_time(ev[1]))
        assert cz.last_status(wsm) == cz.OK
        SL = int(r.out_bytes.item())
        tcm, tdm = float(np.median(tc[1:])) / 1e3, float(np.median(td[1:])) / 1e3
        out[f"32_lorenzo{dims}d"] = {
            "cr": round(4 * n0 / SL, 3),
            "compress_kernel_gbs": round(4 * n0 / tcm / 1e9, 1),
            "decompress_kernel_gbs": round(4 * n0 / tdm / 1e9, 1),
            "compress_frac_of_peak": round((4 * n0 + SL) / tcm / 1e9 / peak, 4),
            "decompress_frac_of_peak": round((4 * n0 + SL) / tdm / 1e9 / peak, 4)}
        del wsm
    del x0
    torch.cuda.empty_cache()
    return out


PAPER_DATASETS = {
    "compress_gbs": {"CESM-ATM": 41.77, "QMCPack": 140.44},
    "decompress_gbs": {"CESM-ATM": 49.91, "NYX": 190.11},
    "source": "PAPER.md P:963-966 (A100, end-to-end, real data, mean over REL 1E-1..1E-4; the other "
              "per-dataset bars of Fig 13 are not legible in the text)"}


def datasets_table(peak: float, steps: int, dev) -> dict:
    """The paper's six datasets (Table 2, one field shape each; synth.DATASETS)
    at REL 1e-2 / 1e-3 / 1e-4: GB/s of fp32 input for REL compression (range +
    compress kernel, the paper's end-to-end compression), decompression, the
    round trip, CR per bound, and each kernel's fraction of the HBM peak;
    L2 flushed before every round trip, every stream's status checked."""
    import synth

    r = Runner(dev, max(280_953_867, 512 ** 3))
    out = {"rel": synth.DATASET_RELS, "unit": "GB/s of fp32 input", "steps": steps}
    for name, spec in synth.DATASETS.items():
        xs = {f: synth.dataset_field(name, f, dev) for f in spec["fields"]}
        jobs = [(f"{f}@{rel:g}", xs[f], xs[f].numel(), rel) for f in spec["fields"] for rel in synth.DATASET_RELS]
        acc, sizes, _, _ = r.measure(jobs, steps, 3)
        d = summarise(jobs, acc, sizes, steps, 1, peak)
        cr = {}
        for rel in synth.DATASET_RELS:
            labs = [f"{f}@{rel:g}" for f in spec["fields"]]
            n_in = sum(4 * xs[f].numel() for f in spec["fields"])
            cr[f"{rel:g}"] = round(n_in / sum(sizes[lab] for lab in labs), 3)     # aggregate over the fields
        out[name] = {"dims_per_field": spec["dims"], "fields": spec["fields"],
                     "n_per_field": [xs[f].numel() for f in spec["fields"]],
                     "compress_gbs": round(d["compress_gbs"], 1), "decompress_gbs": round(d["decompress_gbs"], 1),
                     "round_trip_gbs": round(d["round_trip_gbs"], 1), "cr": cr,
                     "rel_compress_frac_of_peak": round(d["rel_compress_frac_of_peak"], 4),
                     "frac_of_peak": {k: round(v["frac_of_peak"], 4) for k, v in d["kernels"].items()}}
        del xs, jobs
        torch.cuda.empty_cache()
    out["paper_context"] = PAPER_DATASETS
    del r
    torch.cuda.empty_cache()
    return out


def verify(r: Runner, jobs) -> dict:
    """Every job's round trip checked on the device with the fused quality
    kernel (cuszp_quality, untimed): the bound of DESIGN sec 5 and PSNR."""
    cz = r.cz
    q = {"psnr": {}, "max_abs_err_over_eb": {}}
    for lab, x, n, rel in jobs:
        r.round_trip(x, n, rel)
        hdr = cz.read_header(r.out)
        assert hdr["status"] == 0 and cz.last_status(r.ws) == cz.OK
        qv = cz.quality(x, r.y[:n], bound=float(hdr["eb_abs"]), sync=False).cpu()
        ulp_max = float(np.spacing(np.float32(max(abs(qv[0].item()), abs(qv[1].item())))))
        assert qv[3].item() <= hdr["eb_abs"] + ulp_max, (lab, qv[3].item(), hdr["eb_abs"])
        q["psnr"][lab] = round(qv[7].item(), 3)
        q["max_abs_err_over_eb"][lab] = round(qv[3].item() / hdr["eb_abs"], 6)
    return q


def run_ours(args, rank, world, dev):
    import paper_conf_sc_huangd0lc23_b200 as cz

    cfg = resolve_config(args, world)
    fields, rels = config_jobs(cfg)
    group = torch.distributed.group.WORLD if world > 1 else None
    peak, peak_src = peak_hbm()

    # ---- inputs resident in HBM: this rank's block-aligned slab of every field
    xs, n_total = {}, 0
    for f in fields:
        full = make_field(cfg, f, dev)
        n_total += full.numel() * len(rels)
        s0, s1 = slab(full.numel(), rank, world)
        xs[f] = full[s0:s1].clone() if world > 1 else full
        del full
    torch.cuda.empty_cache()
    jobs = [(f"{f}@{rel:g}" if f else f"{rel:g}", xs[f], xs[f].numel(), rel) for f in fields for rel in rels]
    nmax = max(x.numel() for x in xs.values())
    r = Runner(dev, nmax, world, group)
    clocks = ClockSampler(dev.index)
    acc, sizes, wall, clk = r.measure(jobs, args.steps, args.warmup, clocks)
    K = args.steps
    d = summarise(jobs, acc, sizes, K, world, peak, n_total=n_total)
    dom = max(acc, key=acc.get)
    traffic, traffic_src = None, None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as fh:
            js = json.load(fh)
        if js.get("workload") == cfg:
            traffic = js.get("dram_bytes_per_launch", {}).get(dom)
            traffic_src = js.get("source")
    except Exception:
        pass
    achieved = d["kernels"][dom]["algorithmic_gbs"]
    line = {
        "metric": METRIC,
        "value": d["round_trip_gbs"],
        "unit": "GB/s", "n_gpus": world, "steps": K, "warmup": max(args.warmup, 3),
        "ms_per_step": d["ms_per_step"], "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfg, "fields": [f for f in fields if f] or None, "rel": rels,
                   "n_elements": n_total // len(rels),
                   "n_per_rank": [b - a for a, b in (slab(n_total // len(rels) // len(fields), p, world)
                                                     for p in range(world))],
                   "round_trips_per_step": len(jobs),
                   "parallelism": f"sharded x{world} (block-aligned slabs, global range)" if world > 1 else "single",
                   "l2": "inputs > L2; flushed anyway (512 MB write + read, untimed) before every round trip"},
        "compress_gbs": d["compress_gbs"],
        "compress_kernel_only_gbs": d["compress_kernel_only_gbs"],
        "decompress_gbs": d["decompress_gbs"],
        "rel_compress_frac_of_peak": d["rel_compress_frac_of_peak"],
        "cr": d["cr"],
        "kernels": d["kernels"],
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                     "peak_source": peak_src,
                     "algorithmic_bytes_per_launch": d["alg_bytes_per_step"][dom] // len(jobs)},
        "gpu_launches": 3 * len(jobs) * K,
        "clocks": clk,
        "wall_s_timed_region": wall,
        "paper_context": PAPER_A100,
    }
    line["quality"] = verify(r, jobs)

    if not args.no_e2e:
        prev, placement = (bind_to_gpu_numa(dev.index) if os.environ.get("CUSZP_E2E_NUMA", "1") == "1"
                           else (None, "not bound (CUSZP_E2E_NUMA=0)"))
        hx = {}
        h_jobs = [(lab, hx.setdefault(id(x), x.cpu().pin_memory()), rel) for lab, x, _, rel in jobs]
        line["e2e"] = e2e_measure(cz, dev, h_jobs, K, world, r.cap, nmax)
        line["e2e"]["host_placement"] = placement
        del h_jobs, hx
        if prev is not None:
            os.sched_setaffinity(0, prev)        # the CPU baseline may use every core again

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        lab, x, n, rel = jobs[len(jobs) // 2]
        line["cpu_baseline"] = cpu_baseline(x.cpu().numpy(), rel, args.cpu_seconds, f"{cfg}/{lab}")

    del xs, jobs, r
    torch.cuda.empty_cache()
    if world == 1 and not args.no_secondary:
        # every other config at N = 1, each with buffers of its own size
        sec = {"c1_graph": graph_replay_c1(Runner(dev, 1 << 20), max(K, 10), peak)}
        torch.cuda.empty_cache()
        for c, nmax_c in (("c2_hurricane", 25_000_000), ("c4_nyx", 512 ** 3), ("c5_rtm", 1_705_544_460)):
            if c != cfg:
                sec[c] = secondary(Runner(dev, nmax_c), c, 5 if c != "c5_rtm" else 3, peak)
                torch.cuda.empty_cache()
        line["secondary"] = sec
    if world == 1 and not args.no_variants:
        line["block_len_variants"] = variants(Runner(dev, 25_000_000), peak, 5)
        torch.cuda.empty_cache()
    if world == 1 and not args.no_datasets:
        line["datasets"] = datasets_table(peak, 3, dev)
    return line


def bind_to_gpu_numa(dev_index: int):
    """Pin this process to the CPUs local to the GPU (NVML's affinity mask,
    intersected with the CPUs we may use), so pinned host buffers are first
    touched -- and allocated -- on the GPU's NUMA node, as a serving process
    would be placed.  Returns (previous CPU set, description) or (None, why)."""
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
        words = pynvml.nvmlDeviceGetCpuAffinity(h, (os.cpu_count() + 63) // 64)
        local = {64 * i + b for i, w in enumerate(words) for b in range(64) if (int(w) >> b) & 1}
        allowed = os.sched_getaffinity(0)
        cpus = local & allowed
        if not cpus or cpus == allowed:
            return None, f"not bound ({len(local)} GPU-local CPUs, {len(allowed)} allowed)"
        os.sched_setaffinity(0, cpus)
        return allowed, f"bound to the {len(cpus)} GPU-local CPUs of {len(allowed)}"
    except Exception as e:  # no NVML / no affinity support: leave the placement alone
        return None, f"not bound ({type(e).__name__})"


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
