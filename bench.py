#!/usr/bin/env python
"""bench.py -- bulk execution of oblivious algorithms on B200 (libbulkobl).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload ps2|ps2col|ps1|tr1|tr2]
                    [--impl ours|reference] [--no-extras] [--no-cpu-baseline] [--sweep]
                    [--dist-backend nccl|gloo]

--gpus N > 1 without WORLD_SIZE in the environment re-executes this script
under `torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1`
(one rank per GPU); under torchrun the world size must equal N.  --sweep runs
BASELINE configs[4] (p = 2^10..2^22 per rank, both algorithms) instead of the
headline workload.

Headline workload (BASELINE.json configs[1]): bulk prefix sums, fp32, n=1024,
p=2^20 instances PER GPU (weak scaling; rank r owns global instances
[r*p, (r+1)*p)), inputs arriving row-wise (one instance per row) and
processed in the paper's column-wise order with the row<->column
transpose fused on chip (TMA tiles through shared memory).  A step = one
bulk_prefix_sums call over the resident 4 GiB input (out of place, so every
step sees the same data; 4 GiB > 126 MB L2, no flush needed).

One JSON line on rank 0.  Besides the contract keys it carries `roofline`
(dominant kernel vs MEASURED_PEAKS.json HBM), `cpu_baseline` (the oracle on
this host's cores, bounded sample), `e2e` (host pinned buffers through
bulk_prefix_sums_host, H2D + D2H inside the timed region), and `extras`:
the other §8 rows measured the same way (column-wise resident, explicit
transposes, the paper's naive kernel, PS-1 latency, TR-1 and TR-2
triangulation with their rooflines).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

METRIC = "instances/sec at 1/2/4/8 B200; prefix-sum HBM GB/s vs peak"
UNIT = "instances/s"

WORKLOADS = {
    "ps2": dict(seed=2, algo="prefix", n=1024, p=2 ** 20, dtype="float32", layout=0, variant=0,
                desc="bulk prefix-sums fp32 n=1024, p=2^20 per GPU, row-wise in/out, column-wise order with "
                     "the transpose fused on chip (BASELINE configs[1])"),
    "ps2col": dict(seed=2, algo="prefix", n=1024, p=2 ** 20, dtype="float32", layout=1, variant=0,
                   desc="bulk prefix-sums fp32 n=1024, p=2^20 per GPU, column-wise resident"),
    "ps2tr": dict(seed=2, algo="prefix", n=1024, p=2 ** 20, dtype="float32", layout=0, variant=4,
                  desc="bulk prefix-sums fp32 n=1024, p=2^20, row-wise via explicit transpose kernels"),
    "tr_transpose": dict(seed=2, algo="transpose", n=1024, p=2 ** 20, dtype="float32", layout=0, variant=0,
                         desc="SURVEY row a1: layout transpose of the PS-2 data, row-wise [p][n] -> column-wise "
                              "[n][p] (P:120-126)"),
    "ps2naive_col": dict(seed=2, algo="prefix", n=1024, p=2 ** 20, dtype="float32", layout=1, variant=5,
                         desc="the paper's column-wise kernel (thread per instance, 32-bit accesses)"),
    "ps1": dict(seed=1, algo="prefix", n=32, p=1024, dtype="int32", layout=0, variant=0,
                desc="bulk prefix-sums int32 n=32, p=1024 (BASELINE configs[0], latency-bound)"),
    "tr1": dict(seed=3, algo="tri", n=16, p=65536, dtype="int32", layout=0, variant=0,
                desc="bulk optimal triangulation int32 n=16, p=65536 (BASELINE configs[2])"),
    "tr2": dict(seed=4, algo="tri", n=64, p=65536, dtype="float32", layout=0, variant=0,
                desc="bulk optimal triangulation fp32 n=64, p=65536 (BASELINE configs[3])"),
    "tr2col": dict(seed=4, algo="tri", n=64, p=65536, dtype="float32", layout=1, variant=0,
                   desc="TR-2 with the weights in the paper's column-wise arrangement [n][n][p] (P:212)"),
    "tr2umm": dict(seed=4, algo="tri", n=64, p=65536, dtype="float32", layout=1, variant=16,
                   desc="the paper's column-wise UMM kernel on TR-2"),
    "tr1col": dict(seed=3, algo="tri", n=16, p=65536, dtype="int32", layout=1, variant=0,
                   desc="bulk optimal triangulation int32 n=16, p=65536, column-wise weights"),
    "tr1packed": dict(seed=3, algo="tri", n=16, p=65536, dtype="int32", layout=2, variant=0,
                      desc="NEXT-4: TR-1 with packed weights (only the C(n-1,2) weights OPT reads)"),
    "tr2packed": dict(seed=4, algo="tri", n=64, p=65536, dtype="float32", layout=2, variant=0,
                      desc="NEXT-4: TR-2 with packed weights"),
    "tr512": dict(seed=7, algo="tri", n=512, p=1024, dtype="float32", layout=0, variant=0,
                  desc="NEXT-2: the paper's 512-gons at its largest p (P:251), fp32, row-wise"),
    "tr2chords": dict(seed=4, algo="tri", n=64, p=65536, dtype="float32", layout=0, variant="chords",
                      desc="NEXT-1: TR-2 values plus the chords of each optimal triangulation"),
    "exec_bitonic_col": dict(seed=6, algo="exec", prog="bitonic", n=64, p=2 ** 20, dtype="float32", layout=1,
                             variant=0, desc="NEXT-3: generic executor, bitonic sort n=64, column-wise (Thm 2)"),
    "exec_bitonic_row": dict(seed=6, algo="exec", prog="bitonic", n=64, p=2 ** 20, dtype="float32", layout=0,
                             variant=0, desc="NEXT-3: generic executor, bitonic sort n=64, row-wise (Thm 2)"),
    "exec_prefix_col": dict(seed=2, algo="exec", prog="prefix", n=1024, p=2 ** 20, dtype="float32", layout=1,
                            variant=0, desc="NEXT-3: generic executor running Algorithm Prefix-sums, column-wise"),
    "exec_prefix_row": dict(seed=2, algo="exec", prog="prefix", n=1024, p=2 ** 20, dtype="float32", layout=0,
                            variant=0, desc="NEXT-3: generic executor running Algorithm Prefix-sums, row-wise, windowed in shared memory"),
    "exec_bitonic_col_jit": dict(seed=6, algo="exec", prog="bitonic", n=64, p=2 ** 20, dtype="float32", layout=1,
                                 variant=0, jit=True,
                                 desc="NEXT-3: the bitonic sort program compiled to a straight-line kernel (bulk_program_compile), column-wise"),
    "exec_bitonic_row_jit": dict(seed=6, algo="exec", prog="bitonic", n=64, p=2 ** 20, dtype="float32", layout=0,
                                 variant=0, jit=True,
                                 desc="NEXT-3: the bitonic sort program compiled, row-wise (rows staged in shared memory)"),
    "exec_prefix_row_jit": dict(seed=2, algo="exec", prog="prefix", n=1024, p=2 ** 20, dtype="float32", layout=0,
                                variant=0, jit=True,
                                desc="NEXT-3: Algorithm Prefix-sums as a program, compiled (windowed rows), row-wise"),
    "exec_prefix_col_jit": dict(seed=2, algo="exec", prog="prefix", n=1024, p=2 ** 20, dtype="float32", layout=1,
                                variant=0, jit=True,
                                desc="NEXT-3: Algorithm Prefix-sums as a program, compiled (streaming shape), column-wise"),
    # the paper's other experiment shapes (§V): n = 32K floats at p = 8K, 8-gons at
    # p = 4M, our kernels beside the paper's naive row-/column-wise kernels (Figs. 11, 12)
    "ps32k": dict(seed=21, algo="prefix", n=32768, p=8192, dtype="float32", layout=0, variant=0,
                  desc="paper shape: prefix sums of n=32K floats, p=8K (P:249), row-wise, AUTO"),
    "ps32k_col": dict(seed=21, algo="prefix", n=32768, p=8192, dtype="float32", layout=1, variant=0,
                      desc="paper shape: prefix sums n=32K, p=8K, column-wise, AUTO"),
    "ps32k_naive_row": dict(seed=21, algo="prefix", n=32768, p=8192, dtype="float32", layout=0, variant=5,
                            desc="paper shape n=32K, p=8K: the paper's row-wise kernel (Fig. 11)"),
    "ps32k_naive_col": dict(seed=21, algo="prefix", n=32768, p=8192, dtype="float32", layout=1, variant=5,
                            desc="paper shape n=32K, p=8K: the paper's column-wise kernel (Fig. 11)"),
    "tr8": dict(seed=23, algo="tri", n=8, p=4 * 2 ** 20, dtype="float32", layout=0, variant=0,
                desc="paper shape: 8-gons at p=4M (P:251), fp32, row-wise, AUTO"),
    "tr8col": dict(seed=23, algo="tri", n=8, p=4 * 2 ** 20, dtype="float32", layout=1, variant=0,
                   desc="paper shape: 8-gons at p=4M, column-wise weights, AUTO"),
    "tr8_umm_row": dict(seed=23, algo="tri", n=8, p=4 * 2 ** 20, dtype="float32", layout=0, variant=16,
                        desc="paper shape 8-gons p=4M: the paper's row-wise UMM kernel (Fig. 12)"),
    "tr8_umm_col": dict(seed=23, algo="tri", n=8, p=4 * 2 ** 20, dtype="float32", layout=1, variant=16,
                        desc="paper shape 8-gons p=4M: the paper's column-wise UMM kernel (Fig. 12)"),
    "ps2naive_row": dict(seed=2, algo="prefix", n=1024, p=2 ** 20, dtype="float32", layout=0, variant=5,
                         desc="the paper's row-wise kernel (thread per instance, uncoalesced)"),
}
EXTRAS = ["ps2col", "ps2tr", "tr_transpose", "ps1", "tr1", "tr1col", "tr1packed", "tr2", "tr2col", "tr2packed", "tr2chords", "tr512", "ps2naive_col", "ps2naive_row", "tr2umm",
          "exec_bitonic_col", "exec_bitonic_row", "exec_prefix_col", "exec_prefix_row",
          "exec_bitonic_col_jit", "exec_bitonic_row_jit", "exec_prefix_col_jit", "exec_prefix_row_jit",
          "ps32k", "ps32k_col", "ps32k_naive_row", "ps32k_naive_col", "tr8", "tr8col", "tr8_umm_row", "tr8_umm_col"]
# The paper's own fitted GTX Titan models, in ms for p instances: context for the
# extras of the same shape, never a target (another machine, another decade)
PAPER_MODEL_MS = {
    "ps1": ("row-wise 37 us + 8.09 ns * p (n=32, P:249)", lambda p: 0.037 + 8.09e-6 * p),
    "tr8": ("row-wise 0.09 ms + 50.8 ns * p (8-gons, P:251)", lambda p: 0.09 + 50.8e-6 * p),
    "tr8_umm_row": ("row-wise 0.09 ms + 50.8 ns * p (8-gons, P:251)", lambda p: 0.09 + 50.8e-6 * p),
    "tr8col": ("column-wise 0.032 ms + 2.11 ns * p (8-gons, P:260)", lambda p: 0.032 + 2.11e-6 * p),
    "tr8_umm_col": ("column-wise 0.032 ms + 2.11 ns * p (8-gons, P:260)", lambda p: 0.032 + 2.11e-6 * p),
}
L2_BYTES = 126 * 2 ** 20


# ------------------------------------------------------------------ helpers
def comb3(n):
    return n * (n - 1) * (n - 2) // 6


def algo_bytes_per_instance(wl):
    """Algorithmic HBM bytes per instance: prefix reads
    and writes n elements; OPT reads the C(n-1,2) weights c[a][b], b-a>=2
    (the only ones Algorithm OPT touches) and writes one result."""
    if wl["algo"] in ("prefix", "exec", "transpose"):
        return 2 * wl["n"] * 4
    n = wl["n"]
    return 4 * ((n - 1) * (n - 2) // 2 + 1)


def addmin_per_instance(wl):
    return comb3(wl["n"]) if wl["algo"] == "tri" else 0


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d, "measured (MEASURED_PEAKS.json)"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback (B200_PROFILING.md)"


def load_traffic():
    path = os.path.join(ROOT, "profiles", "traffic.json")   # workload -> ncu DRAM bytes per launch
    try:
        with open(path) as f:
            return json.load(f)
    except Exception:
        return {}


class ClockSampler:
    """Polls NVML every few ms while the timed region runs."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.reasons = set()
        self._stop = threading.Event()
        self.ok = False
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.ok = False

    def _run(self):
        nv = self.nv
        names = {
            "gpu_idle": getattr(nv, "nvmlClocksEventReasonGpuIdle", 0x1),
            "applications_clocks_setting": getattr(nv, "nvmlClocksEventReasonApplicationsClocksSetting", 0x2),
            "sw_power_cap": getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4),
            "hw_slowdown": getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8),
            "sync_boost": getattr(nv, "nvmlClocksEventReasonSyncBoost", 0x10),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
            "hw_power_brake_slowdown": getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                try:
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                except Exception:
                    r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for k, bit in names.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": len(self.samples)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def _free_port():
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    return port


def self_launch_argv(gpus, argv, port):
    """The torchrun command line `--gpus N` (N > 1, no WORLD_SIZE set) re-executes
    bench.py under: one rank per GPU, rendezvous on 127.0.0.1."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
            "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *argv]


def maybe_self_launch(args, argv):
    """Returns None when this process is a rank to run; else the exit code of the
    torchrun child this process spawned for `--gpus N`."""
    if args.gpus is None or args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    if args.impl == "reference":          # the CPU arm: rank 0 alone does work
        return None
    import subprocess
    return subprocess.call(self_launch_argv(args.gpus, argv, _free_port()))


class Ctx:
    def __init__(self, backend="nccl"):
        self.rank = int(os.environ.get("RANK", 0))
        self.world = int(os.environ.get("WORLD_SIZE", 1))
        self.local = int(os.environ.get("LOCAL_RANK", 0))
        self.dist = self.world > 1
        self.backend = backend
        # one process per GPU; the modulo only matters for the gloo test mode
        # (several ranks sharing one GPU to exercise the multi-rank logic)
        self.device = self.local % max(1, torch.cuda.device_count()) if torch.cuda.is_available() else 0

    def barrier(self):
        if self.dist:
            if self.backend == "nccl":
                dist.barrier(device_ids=[self.device])
            else:
                dist.barrier()

    def max(self, x: float) -> float:
        from paper_conf_ipps_tanitni14_b200 import shard
        return shard.max_over_ranks(x)


def timed(ctx, fn, steps, warmup, stream):
    """Average device ms per step (CUDA events on `stream` around all K steps),
    max over ranks, plus the number of libbulkobl kernel launches inside the
    timed region.  Inputs are never L2-resident: a step's input either exceeds
    2x L2 or is one of enough rotating copies (copies_for)."""
    import paper_conf_ipps_tanitni14_b200 as bo
    with torch.cuda.stream(stream):
        for _ in range(warmup):
            fn()
    torch.cuda.synchronize()
    ctx.barrier()
    torch.cuda.synchronize()
    launches0 = bo.launch_count()
    # A spin kernel ahead of the timed region lets the host queue every step
    # before the GPU reaches the first event, so small kernels are not timed
    # with host launch gaps between them (it runs before the first event).
    with torch.cuda.stream(stream):
        torch.cuda._sleep(int(min(steps * 200e-6, 0.05) * 2.0e9))
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        ev0.record(stream)
        for _ in range(steps):
            fn()
        ev1.record(stream)
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / steps
    launches = bo.launch_count() - launches0
    ctx.barrier()
    return ctx.max(ms), launches


# ------------------------------------------------------------ our arm
def copies_for(wl):
    """Input copies a step rotates through: 1 when one input exceeds 2x L2, else
    enough that the copies together exceed 2x L2, so no step reads an input
    that is still L2-resident (the timing rule's alternative to a flush)."""
    b = input_bytes(wl)
    return 1 if b >= 2 * L2_BYTES else min(4096, -(-2 * L2_BYTES // b) + 1)


def _rotator(x, copies):
    xs = [x] + [x.clone() for _ in range(copies - 1)]
    i = [0]

    def nxt():
        v = xs[i[0]]
        i[0] = (i[0] + 1) % len(xs)
        return v
    return nxt


def l2_note(wl, copies):
    if copies == 1:
        return f"input {input_bytes(wl) / 2 ** 30:.2f} GiB per GPU > 2x the 126 MB L2; no flush needed"
    return (f"input {input_bytes(wl) / 2 ** 20:.2f} MiB < 2x L2: steps rotate over {copies} copies "
            f"({copies * input_bytes(wl) / 2 ** 20:.0f} MiB > 2x the 126 MB L2), so no step reads an L2-resident input")


def setup_workload(wl, rank, copies=1):
    import paper_conf_ipps_tanitni14_b200 as bo
    n, p = wl["n"], wl["p"]
    dt = getattr(torch, wl["dtype"])
    from paper_conf_ipps_tanitni14_b200 import shard
    h0, _ = shard.weak_range(p, rank)
    seed = wl["seed"]
    if wl["algo"] == "exec":
        from paper_conf_ipps_tanitni14_b200 import programs
        prog = programs.bitonic_sort(n) if wl["prog"] == "bitonic" else programs.prefix_sums(n, wl["dtype"])
        x = bo.generate_prefix(n, p, seed, dt, wl["layout"], "uniform", h0=h0)
        prep = bo.prepare(prog, n)          # validated, rewritten and uploaded once, outside the timed steps
        how = "prepared"
        if wl.get("jit"):                   # NVRTC-compiled straight-line kernel, built outside the timed steps
            how = "compiled" if prep.compile(dt, wl["layout"]) else "prepared (not compiled)"
        nxt = _rotator(x, copies)

        def fn():
            bo.execute(prep, nxt(), wl["layout"])
        return dict(x=x, out=x, fn=fn, seed=seed, h0=h0, prep=prep,
                    variant=f"exec[{wl['prog']}: {prog.array().shape[0]} instr, {how}]")
    if wl["algo"] == "transpose":
        x = bo.generate_prefix(n, p, seed, dt, bo.ROW_WISE, "uniform", h0=h0)        # [p][n]
        out = torch.empty((n, p), dtype=dt, device="cuda")
        nxt = _rotator(x, copies)

        def fn():
            bo.transpose(nxt(), out=out)
        return dict(x=x, out=out, fn=fn, seed=seed, h0=h0, variant="transpose_tma")
    if wl["algo"] == "prefix":
        x = bo.generate_prefix(n, p, seed, dt, wl["layout"], "uniform", h0=h0)
        out = torch.empty_like(x)
        ws = None
        need = bo.prefix_sums_workspace(n, p, bo.F32 if wl["dtype"] == "float32" else bo.I32, wl["layout"],
                                        wl["variant"])
        if need:
            ws = torch.empty(need, dtype=torch.uint8, device="cuda")

        nxt = _rotator(x, copies)

        def fn_on(src):
            bo.prefix_sums(src, wl["layout"], wl["variant"], out=out, workspace=ws)

        def fn():
            fn_on(nxt())
        variant = bo.prefix_sums_variant(n, p, bo.F32 if wl["dtype"] == "float32" else bo.I32, wl["layout"],
                                         wl["variant"])
    else:
        x = bo.generate_tri(n, p, seed, dt, wl["layout"], h0=h0)
        out = torch.empty(p, dtype=dt, device="cuda")
        dcode = bo.F32 if wl["dtype"] == "float32" else bo.I32
        nxt = _rotator(x, copies)
        if wl["variant"] == "chords":
            def fn():
                bo.triangulation_chords(nxt(), wl["layout"])
            return dict(x=x, out=out, fn=fn, seed=seed, h0=h0, variant="tiled_half+chords")
        need = bo.triangulation_workspace(n, p, dcode, wl["layout"], wl["variant"])
        ws = torch.empty(need, dtype=torch.uint8, device="cuda") if need else None

        def fn_on(src):
            bo.triangulation(src, wl["layout"], wl["variant"], out=out, workspace=ws)

        def fn():
            fn_on(nxt())
        variant = bo.triangulation_variant(n, p, dcode, wl["layout"], wl["variant"])
    return dict(x=x, out=out, fn=fn, fn_on=fn_on, seed=seed, h0=h0,
                variant=bo.VARIANT_NAMES.get(variant, str(variant)))


def input_bytes(wl):
    n, p = wl["n"], wl["p"]
    if wl["algo"] in ("prefix", "exec", "transpose"):
        return n * p * 4
    return ((n - 1) * (n - 2) // 2 if wl["layout"] >= 2 else n * n) * p * 4


def measure(ctx, name, steps, warmup, stream, peaks, traffic):
    wl = WORKLOADS[name]
    copies = copies_for(wl)
    st = setup_workload(wl, ctx.rank, copies)
    ms, launches = timed(ctx, st["fn"], steps, warmup, stream)
    p_all = wl["p"] * ctx.world
    res = {"desc": wl["desc"], "variant": st["variant"], "n": wl["n"], "p_per_gpu": wl["p"],
           "dtype": wl["dtype"], "layout": "row-wise" if wl["layout"] == 0 else "column-wise",
           "ms_per_step": ms, "value": p_all / (ms * 1e-3), "unit": UNIT,
           "l2": l2_note(wl, copies),
           "gpu_launches": launches}
    bytes_launch = algo_bytes_per_instance(wl) * wl["p"]
    if wl["algo"] in ("prefix", "exec", "transpose"):
        gbs = bytes_launch / (ms * 1e-3) / 1e9
        res["algorithmic_GBps_per_gpu"] = gbs
        res["roofline"] = {"bound": "hbm", "achieved": gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                           "frac": gbs / peaks["hbm_gbs"], "traffic": traffic.get(name, {}).get("dram_bytes_per_launch")}
    else:
        res["roofline"] = tri_roofline(wl, ms * steps / max(1, launches), peaks)
    if name in PAPER_MODEL_MS:
        what, model = PAPER_MODEL_MS[name]
        res["paper_gtx_titan_model"] = {"ms_per_step": model(wl["p"]), "model": what,
                                        "note": "the paper's fitted model on its GTX Titan: context, not a target"}
    return res, st


def tri_roofline(wl, per_launch_ms, peaks):
    """Triangulation is bounded by whichever roof is slower for its work
    (SURVEY.md §8 d): HBM for the algorithmic bytes or the ALU for the C(n,3)
    add-mins.  Returns the binding roof, with the other one alongside."""
    p = wl["p"]
    secs = per_launch_ms * 1e-3
    gbs = algo_bytes_per_instance(wl) * p / secs / 1e9
    tops = addmin_per_instance(wl) * p / secs / 1e12
    alu = alu_peak_taddmin(peaks, wl["dtype"])
    hbm = {"bound": "hbm", "achieved": gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": gbs / peaks["hbm_gbs"]}
    alu_r = {"bound": "alu", "achieved": tops, "peak": alu, "unit": "T add-min/s", "frac": tops / alu,
             "peak_source": "measured, profiles/r02/addmin_peak.json (tools/micro/addmin_peak.cu: single-pipe probes at 99 % pipe utilisation)"}
    t_hbm = algo_bytes_per_instance(wl) * p / (peaks["hbm_gbs"] * 1e9)
    t_alu = addmin_per_instance(wl) * p / (alu * 1e12)
    main, other = (hbm, alu_r) if t_hbm >= t_alu else (alu_r, hbm)
    out = dict(main)
    out["other_roof"] = other
    out["roof_time_us"] = {"hbm": t_hbm * 1e6, "alu": t_alu * 1e6}
    return out


ADDMIN_PEAK_JSON = os.path.join(ROOT, "profiles", "r02", "addmin_peak.json")


def alu_peak_taddmin(peaks, dtype):
    """ALU roof for the min-plus inner step, MEASURED (SURVEY §8 d): read from the
    committed profiles/r02/addmin_peak.json (tools/micro/addmin_peak.cu on B200):
    fp32 -- the slower of FADD2 alone (FMA pipe at 99.5 %) and FMNMX3 alone (ALU
    pipe at 98.9 %), 121.9 add-mins per SM-clock; int32 -- the fastest measured
    form, 71.0.  Scaled by 148 SMs and the max SM clock."""
    with open(ADDMIN_PEAK_JSON) as fh:
        d = json.load(fh)
    per_sm_clk = d["fp32" if dtype == "float32" else "int32"]["roof_per_sm_clk"]
    mhz = peaks.get("sm_max_mhz", 1965.0)
    return d["sm_count"] * per_sm_clk * mhz * 1e6 / 1e12


def cpu_baseline(ctx, name, st, budget_s=12.0):
    """The oracle as it stands on this host's cores, on a bounded sample of the
    same workload; also checks the GPU outputs of the sampled instances."""
    import bulkgen
    import oracle
    wl = WORKLOADS[name]
    n, p = wl["n"], wl["p"]
    cores = os.cpu_count() or 1

    def inputs(ids):
        if wl["algo"] == "prefix":
            return bulkgen.prefix_instances(n, ids, st["seed"], wl["dtype"])
        return bulkgen.tri_instances(n, ids, st["seed"], wl["dtype"])

    def run(x, threads=cores):
        if wl["algo"] == "prefix":
            return oracle.bulk_prefix_sums(x, oracle.ROW_WISE, nthreads=threads)
        return oracle.bulk_opt(x, oracle.ROW_WISE, nthreads=threads)

    # calibrate
    k = 256
    while True:
        ids = np.arange(st["h0"], st["h0"] + k)
        x = inputs(ids)
        t0 = time.perf_counter()
        run(x)
        dt = time.perf_counter() - t0
        if dt > 0.5 or k >= p:
            break
        k = min(p, k * 8)
    rate = k / dt
    k = int(min(p, max(k, rate * budget_s)))
    # sample = evenly spaced instances across the rank's shard
    ids = np.unique(np.linspace(st["h0"], st["h0"] + p - 1, k).astype(np.int64))
    x = inputs(ids)
    t0 = time.perf_counter()
    ref = run(x)
    dt = time.perf_counter() - t0
    reps = 1
    if dt < 2.0:                             # whole workload in well under 2 s: time repeated passes
        reps = int(min(512, max(2, 2.0 / max(dt, 1e-6))))
        t0 = time.perf_counter()
        for _ in range(reps):
            run(x)
        dt = (time.perf_counter() - t0) / reps
    # one core, like the paper's single-CPU baseline: a ~2 s sample
    k1 = max(32, min(len(ids), int(2.0 * len(ids) / max(dt * cores, 1e-9))))
    x1 = x[:k1]
    t0 = time.perf_counter()
    run(x1, threads=1)
    dt1 = time.perf_counter() - t0
    # parity of the sampled instances (GPU output vs oracle)
    loc = torch.from_numpy(ids - st["h0"]).cuda()
    out = st["out"]
    if wl["algo"] == "prefix":
        g = out[loc] if wl["layout"] == 0 else out[:, loc].T
    else:
        g = out[loc]
    g = g.contiguous().cpu().numpy()
    ok = bool(np.array_equal(g.view(np.uint32), ref.view(np.uint32)))
    return {"value": len(ids) / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{len(ids)} of the {p} instances of workload '{name}' (evenly spaced ids), "
                      f"plain C oracle, {cores} threads, {dt:.3f} s per pass"
                      + (f" (mean of {reps} passes)" if reps > 1 else ""),
            "single_core": {"value": k1 / dt1, "unit": UNIT, "cores": 1,
                            "sample": f"first {k1} instances of the sample, {dt1:.2f} s"},
            "cpu_model": cpu_model(),
            "gpu_matches_oracle_on_sample": ok}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def e2e(ctx, name, steps, warmup):
    """Same metric through the public host-buffer API: pinned host input, H2D,
    kernels and D2H inside the timed region (library pipelines chunks)."""
    import paper_conf_ipps_tanitni14_b200 as bo
    wl = WORKLOADS[name]
    n, p = wl["n"], wl["p"]
    dt = getattr(torch, wl["dtype"])
    if wl["algo"] not in ("prefix", "tri"):
        return None
    tri = wl["algo"] == "tri"
    dcode = bo.F32 if wl["dtype"] == "float32" else bo.I32
    err = None
    try:
        if tri:
            dev = bo.generate_tri(n, p, wl["seed"], dt, wl["layout"], h0=ctx.rank * p)
            in_bytes, out_bytes = dev.numel() * 4, p * 4
            need = bo.triangulation_host_bytes(n, p, dcode, wl["layout"], wl["variant"])
            h_out = torch.empty(p, dtype=dt, pin_memory=True)
        else:
            dev = bo.generate_prefix(n, p, wl["seed"], dt, wl["layout"], "uniform", h0=ctx.rank * p)
            in_bytes = out_bytes = n * p * 4
            need = bo.prefix_sums_host_bytes(n, p, dcode, wl["layout"], wl["variant"])
            h_out = torch.empty(dev.shape, dtype=dt, pin_memory=True)
        h_in = torch.empty(dev.shape, dtype=dt, pin_memory=True)
        h_in.copy_(dev)
        del dev
        dbuf = torch.empty(need, dtype=torch.uint8, device="cuda")
        torch.cuda.synchronize()
    except Exception as exc:        # agree across ranks before any barrier
        err = repr(exc)
    if ctx.max(1.0 if err else 0.0) > 0:
        raise RuntimeError(err or "e2e buffers could not be allocated on another rank")
    stream = torch.cuda.current_stream()

    def fn():
        if tri:
            bo.triangulation_host(h_in, wl["layout"], wl["variant"], out_host=h_out, device_buf=dbuf, stream=stream)
        else:
            bo.prefix_sums_host(h_in, wl["layout"], wl["variant"], out_host=h_out, device_buf=dbuf, stream=stream)
    for _ in range(warmup):
        fn()
    ctx.barrier()
    c0 = bo.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    ev0.record(stream)
    for _ in range(steps):
        fn()
    ev1.record(stream)
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / steps
    ms = ctx.max(ev0.elapsed_time(ev1) / steps)
    ctx.barrier()
    api = "bulk_triangulation_host" if tri else "bulk_prefix_sums_host"
    return {"value": p * ctx.world / (ms * 1e-3), "unit": UNIT, "h2d_bytes_per_step": in_bytes,
            "d2h_bytes_per_step": out_bytes, "ms_per_step": ms, "wall_ms_per_step": wall * 1e3,
            "api": f"{api} (pinned host in/out, 2-stream chunked H2D/compute/D2H)",
            "gpu_launches": bo.launch_count() - c0}


def single_gpu_checksums(wl, st, world):
    """Per-shard checksums of the whole problem computed on THIS GPU alone: shard r
    (global ids [r*p, (r+1)*p)) is regenerated into rank 0's input buffer and run
    with the same call, one shard after the other.  Equal to the all-gathered
    per-rank checksums iff the multi-rank run computed what one GPU computes."""
    import paper_conf_ipps_tanitni14_b200 as bo
    n, p = wl["n"], wl["p"]
    dt = getattr(torch, wl["dtype"])
    x, out = st["x"], st["out"]
    res = []
    for r in range(world):
        h0 = r * p
        if wl["algo"] == "prefix":
            bo.generate_prefix(n, p, wl["seed"], dt, wl["layout"], "uniform", h0=h0, out=x)
        elif wl["algo"] == "tri":
            bo.generate_tri(n, p, wl["seed"], dt, wl["layout"], h0=h0, out=x)
        else:
            return []
        st["fn_on"](x)
        cs = bo.checksum(out, wl["layout"] if wl["algo"] == "prefix" else 0, h0=h0)
        res.append(int(cs.cpu().numpy().view(np.uint64)[0]))
    # leave rank 0's own shard in place again
    if world > 1:
        if wl["algo"] == "prefix":
            bo.generate_prefix(n, p, wl["seed"], dt, wl["layout"], "uniform", h0=st["h0"], out=x)
        else:
            bo.generate_tri(n, p, wl["seed"], dt, wl["layout"], h0=st["h0"], out=x)
        st["fn_on"](x)
    torch.cuda.synchronize()
    return res


def run_ours(args, ctx):
    import paper_conf_ipps_tanitni14_b200 as bo
    bo.lib()
    peaks, peak_src = load_peaks()
    traffic = load_traffic()
    stream = torch.cuda.Stream()
    name = args.workload
    sampler = ClockSampler(ctx.device)
    # primary, with clocks sampled during its timed region
    wl = WORKLOADS[name]
    copies = copies_for(wl)
    st = setup_workload(wl, ctx.rank, copies)
    l2note = l2_note(wl, copies)
    with sampler:
        ms, launches = timed(ctx, st["fn"], args.steps, args.warmup, stream)
    p_all = wl["p"] * ctx.world
    value = p_all / (ms * 1e-3)
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ctx.world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32" if wl["dtype"] == "float32" else "i32", "data": "synthetic",
            "config": {"workload": wl["desc"], "n": wl["n"], "p_per_gpu": wl["p"], "p_total": p_all,
                       "layout_in_out": "row-wise" if wl["layout"] == 0 else "column-wise",
                       "variant": st["variant"], "parallelism": f"instances sharded over {ctx.world} GPU(s)",
                       "l2": l2note,
                       "input": "counter-based synthetic, generated on device from global instance ids"},
            "gpu_launches": launches}
    # roofline of the dominant kernel (the only kernel of the step for AUTO)
    per_launch_ms = ms * args.steps / max(1, launches)
    bytes_launch = algo_bytes_per_instance(wl) * wl["p"]
    if wl["algo"] in ("prefix", "exec"):
        ach = bytes_launch / (per_launch_ms * 1e-3) / 1e9
        tr = traffic.get(name, {}).get("dram_bytes_per_launch")
        line["roofline"] = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                            "frac": ach / peaks["hbm_gbs"], "traffic": tr,
                            "peak_source": peak_src + " hbm_gbs (burst copy)",
                            "kernel": st["variant"], "algorithmic_bytes_per_launch": bytes_launch}
    else:
        line["roofline"] = tri_roofline(wl, per_launch_ms, peaks)
        line["roofline"]["traffic"] = traffic.get(name, {}).get("dram_bytes_per_launch")
        line["roofline"]["kernel"] = st["variant"]
        line["roofline"]["algorithmic_bytes_per_launch"] = algo_bytes_per_instance(wl) * wl["p"]
        line["roofline"]["addmin_per_launch"] = addmin_per_instance(wl) * wl["p"]
    line["clocks"] = sampler.summary()
    # checksum of each rank's shard, one NCCL all-gather (SURVEY §8 e), off the timed region
    from paper_conf_ipps_tanitni14_b200 import shard
    cs = bo.checksum(st["out"], wl["layout"] if wl["algo"] == "prefix" else 0, h0=st["h0"])
    cs_list = shard.gather_checksums(int(cs.cpu().numpy().view(np.uint64)[0]))
    line["checksums"] = {"per_rank": [hex(c) for c in cs_list],
                         "combined": hex(shard.combine_checksums(cs_list)),
                         "note": "one all-gather after the timed region; inputs are generated per rank "
                                 "from global instance ids, so nothing crosses NVLink on the data path"}
    # the oracle on a sample of rank 0's shard (before anything reuses st's buffers)
    if args.cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(ctx, name, st) if ctx.rank == 0 else None
        cb = line["cpu_baseline"]
        if cb and cb.get("single_core"):
            # north_star: quote the paper's GPU-over-one-CPU factor as context only
            line["speedup_context"] = {
                "gpu_over_oracle_one_core": line["value"] / cb["single_core"]["value"],
                "gpu_over_oracle_all_cores": line["value"] / cb["value"],
                "paper": "more than 150x GPU (GTX Titan) over one Core i7 core at n=1K, p>=8K (P:249); "
                         "context only -- another GPU, another CPU, another decade"}
    # G-invariance: rank 0 recomputes every rank's shard on its own GPU, one after
    # the other (what a single-GPU run of the whole problem computes), and compares
    if ctx.rank == 0 and wl["algo"] in ("prefix", "tri") and "fn_on" in st:
        single = single_gpu_checksums(wl, st, ctx.world)
        line["checksums"]["single_gpu_recompute"] = [hex(c) for c in single]
        line["checksums_match"] = single == cs_list
        if "cpu_baseline" in line and line["cpu_baseline"]:
            line["checksums_match_oracle_sample"] = line["cpu_baseline"]["gpu_matches_oracle_on_sample"]
    ctx.barrier()
    if args.extras:
        ex = {}
        for e in EXTRAS:
            if e == name:
                continue
            try:
                r, est = measure(ctx, e, max(5, min(args.steps, 20)), max(3, args.warmup), stream, peaks, traffic)
                ex[e] = r
                del est
            except Exception as exc:  # report, do not hide
                ex[e] = {"error": repr(exc)}
            torch.cuda.empty_cache()
        line["extras"] = ex
    if args.e2e:
        try:
            line["e2e"] = e2e(ctx, name, max(2, min(args.steps, 5)), 1)
        except Exception as exc:                    # e.g. pinned host memory exhausted at 8 ranks
            line["e2e"] = {"error": repr(exc)}
    if ctx.rank == 0:
        print(json.dumps(line), flush=True)


# ------------------------------------------------------------ p-sweep
SWEEP_CASES = [("prefix", 32, "int32", 1), ("prefix", 1024, "float32", 2), ("tri", 16, "int32", 3),
               ("tri", 64, "float32", 4)]


def run_sweep(args, ctx):
    """BASELINE configs[4]: p = 2^lo..2^hi instances PER RANK (weak scaling) for
    both algorithms at the configs' n and dtype, AUTO variant, row-wise inputs,
    timed like the headline (max over ranks).  Every point all-gathers the shard
    checksums, compares them with rank 0's single-GPU recomputation of every
    shard, and checks sampled instances of rank 0's shard against the oracle."""
    import bulkgen
    import oracle
    import paper_conf_ipps_tanitni14_b200 as bo
    from paper_conf_ipps_tanitni14_b200 import shard
    bo.lib()
    lo, hi, step = (int(v) for v in args.sweep_log2.split(":"))
    peaks, _ = load_peaks()
    stream = torch.cuda.Stream()
    points = []
    sampler = ClockSampler(ctx.device)
    with sampler:
        for algo, n, dt, seed in SWEEP_CASES:
            for lg in range(lo, hi + 1, step):
                p = 2 ** lg
                wl = dict(seed=seed, algo=algo, n=n, p=p, dtype=dt, layout=0, variant=0, desc="sweep")
                st = setup_workload(wl, ctx.rank, copies_for(wl))
                ms, launches = timed(ctx, st["fn"], max(5, min(args.steps, 20)), args.warmup, stream)
                st["fn_on"](st["x"])
                cs = bo.checksum(st["out"], 0, h0=st["h0"])
                parts = shard.gather_checksums(int(cs.cpu().numpy().view(np.uint64)[0]))
                pt = {"algo": algo, "n": n, "dtype": dt, "p_per_gpu": p, "p_total": p * ctx.world,
                      "variant": st["variant"], "ms_per_step": ms, "value": p * ctx.world / (ms * 1e-3),
                      "unit": UNIT, "gpu_launches": launches}
                if algo == "prefix":
                    gbs = algo_bytes_per_instance(wl) * p / (ms * 1e-3) / 1e9
                    pt["GBps_per_gpu"] = gbs
                    pt["hbm_frac"] = gbs / peaks["hbm_gbs"]
                else:
                    pt["T_addmin_per_gpu"] = addmin_per_instance(wl) * p / (ms * 1e-3) / 1e12
                if ctx.rank == 0:
                    single = single_gpu_checksums(wl, st, ctx.world)
                    pt["checksums_match"] = single == parts
                    rng = np.random.default_rng(lg)
                    loc = np.unique(np.r_[rng.integers(0, p, 6), 0, p - 1])
                    ids = loc + st["h0"]
                    if algo == "prefix":
                        ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, seed, dt), oracle.ROW_WISE)
                    else:
                        ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, seed, dt), oracle.ROW_WISE)
                    got = st["out"][torch.from_numpy(loc).cuda()].cpu().numpy()
                    pt["oracle_sample_match"] = bool(np.array_equal(np.ascontiguousarray(got).view(np.uint32),
                                                                    ref.view(np.uint32)))
                ctx.barrier()
                points.append(pt)
                del st
                torch.cuda.empty_cache()
    if ctx.rank == 0:
        line = {"mode": "sweep", "metric": METRIC, "unit": UNIT, "n_gpus": ctx.world, "scaling": "weak",
                "higher_is_better": True, "data": "synthetic", "steps": max(5, min(args.steps, 20)),
                "warmup": args.warmup,
                "config": {"workload": "BASELINE configs[4]: p-sweep per GPU, both algorithms, AUTO variants",
                           "log2_p": [lo, hi, step]},
                "all_checksums_match": all(pt.get("checksums_match", True) for pt in points),
                "all_oracle_samples_match": all(pt.get("oracle_sample_match", True) for pt in points),
                "clocks": sampler.summary(), "points": points}
        print(json.dumps(line), flush=True)


# ------------------------------------------------------ reference arm
def run_reference(args, ctx):
    """The paper has no code; the reference arm is the CPU oracle as it stands
    (plain per-instance C loops, Algorithm Prefix-sums / Algorithm OPT) on this
    host's cores, each step a bounded sample of the same workload."""
    if ctx.rank != 0:
        return
    import bulkgen
    import oracle
    wl = WORKLOADS[args.workload]
    n, p = wl["n"], wl["p"]
    cores = os.cpu_count() or 1

    def make(k, off):
        ids = np.arange(off, off + k) % p
        if wl["algo"] == "prefix":
            return bulkgen.prefix_instances(n, ids, wl["seed"], wl["dtype"])
        return bulkgen.tri_instances(n, ids, wl["seed"], wl["dtype"])

    def run(x, threads=cores):
        if wl["algo"] == "prefix":
            return oracle.bulk_prefix_sums(x, oracle.ROW_WISE, nthreads=threads)
        return oracle.bulk_opt(x, oracle.ROW_WISE, nthreads=threads)

    k = 1024
    while True:
        x = make(k, 0)
        t0 = time.perf_counter()
        run(x)
        dt = time.perf_counter() - t0
        if dt > 0.2 or k >= p:
            break
        k = min(p, k * 4)
    per_step_target = min(4.0, 120.0 / max(1, args.steps + args.warmup))
    k = int(min(p, max(256, k / dt * per_step_target)))
    xs = make(k, 0)
    for _ in range(args.warmup):
        run(xs)
    times = []
    for s in range(args.steps):
        t0 = time.perf_counter()
        run(xs)
        times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    value = k / (ms * 1e-3)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ctx.world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32" if wl["dtype"] == "float32" else "i32",
            "data": "synthetic",
            "config": {"workload": wl["desc"], "n": n, "p_per_gpu": p, "sample_instances_per_step": k},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"{k} of {p} instances per step, plain C oracle, {cores} threads"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=None,
                    help="ranks (one per GPU); default: WORLD_SIZE under torchrun, else 1")
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="ps2", choices=sorted(k for k in WORKLOADS if WORKLOADS[k]["algo"] != "transpose"))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-extras", dest="extras", action="store_false")
    ap.add_argument("--no-e2e", dest="e2e", action="store_false")
    ap.add_argument("--no-cpu-baseline", dest="cpu_baseline", action="store_false")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo only to test the multi-rank logic with several ranks on one GPU")
    ap.add_argument("--sweep", action="store_true", help="BASELINE configs[4]: p = 2^10..2^22 per rank")
    ap.add_argument("--sweep-log2", default="10:22:2", help="lo:hi:step of log2(p) for --sweep")
    args = ap.parse_args(argv)
    if args.warmup < 3:
        args.warmup = 3
    rc = maybe_self_launch(args, sys.argv[1:] if argv is None else argv)
    if rc is not None:
        sys.exit(rc)
    ctx = Ctx(args.dist_backend)
    if args.impl == "reference":
        if args.gpus and not ctx.dist:
            ctx.world = args.gpus                # reported; the CPU arm's work does not depend on it
        run_reference(args, ctx)
        return
    if args.gpus is not None and args.gpus != ctx.world:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ctx.world}")
    if ctx.dist and ctx.backend == "nccl" and torch.cuda.device_count() < ctx.world:
        raise SystemExit(f"bench.py: {ctx.world} NCCL ranks need {ctx.world} GPUs, this node has "
                         f"{torch.cuda.device_count()} (use --dist-backend gloo to test the multi-rank "
                         "logic with several ranks per GPU)")
    torch.cuda.set_device(ctx.device)
    if ctx.dist:
        if ctx.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", ctx.device))
        else:
            dist.init_process_group(ctx.backend)
    try:
        if args.sweep:
            run_sweep(args, ctx)
        else:
            run_ours(args, ctx)
    finally:
        if ctx.dist:
            ctx.barrier()
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
