#!/usr/bin/env python3
"""DEFCON hot-path benchmark on B200 (contract: one JSON line from rank 0).

Default workload (BASELINE.json configs[2], the north-star target): YOLACT++ ResNet-101 C4
DCNv2 3x3 layer, N=16 images per GPU, C=256, 35x35, offset_groups=1, bf16 storage, fed by the
paper's lightweight depthwise offset branch.  One "step" = one pass of the whole
hot path over one batch: defcon_offset_dw_conv (step 1) + defcon_dcn_forward (step 2).

--workload picks another BASELINE.json config: c3, c4_g4, c5 (bf16), c4_f32 / c4_g4_f32 (fp32 on
the tensor cores, 3xTF32), c4_f32_simt (the CUDA-core fp32 anchor), or stack -- config 5, the
11-layer interval-placed DCN stack of YOLACT++ R101 C3-C5 at a GLOBAL batch of 64 images
sharded over the GPUs (strong scaling: 64/N images per GPU); a step is then the whole stack.

metric: contraction TFLOP/s (2*M*Cout*K^2*Cin per layer), higher is better;
ms_per_step gives the layer (stack) latency.  value = FLOPs of all ranks / max-over-ranks time.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl reference]
Multi-GPU: launched by torchrun (one rank per GPU, NCCL, images sharded, no data-path
collective).
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

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from defcon_workloads import configs, inputs, sharding  # noqa: E402

# name -> (layers at the per-GPU batch of a 1-GPU run, fp32 mode, strong scaling)
WORKLOADS = {
    "c4": ([configs.C4], "simt", False),
    "c3": ([configs.C3], "simt", False),
    "c4_g4": ([configs.C4_G4], "simt", False),
    "c5": ([configs.C5], "simt", False),
    "c4_f32": ([configs.C4_F32], "3xtf32", False),
    "c4_g4_f32": ([configs.C4_G4_F32], "3xtf32", False),
    "c4_f32_simt": ([configs.C4_F32], "simt", False),
    "stack": (configs.stack_layers(64), "simt", True),
}
STACK_GLOBAL_BATCH = 64
L2_BYTES = 126 * 2**20
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
NCU_SUMMARY_GLOB = os.path.join(ROOT, "profiles", "r*_ncu_summary.json")


def metric_name(name="c4"):
    if name == "stack":
        return ("DEFCON interval-placed DCN stack (11 DCNv2 layers, YOLACT++ R101 C3-C5) TFLOP/s "
                "(contraction) at global batch 64, incl. offset branches")
    c = WORKLOADS[name][0][0]
    shape = {"yolact_r101_c3_v2": "C3", "yolact_r101_c4_v2": "C4", "yolact_r101_c4_v2_g4": "C4 G=4",
             "yolact_r101_c5_v2": "C5", "yolact_r101_c4_v2_f32": "C4 fp32",
             "yolact_r101_c4_v2_g4_f32": "C4 G=4 fp32"}[c.name]
    return f"DCNv2 layer TFLOP/s (contraction) at YOLACT++ {shape} shape, incl. offset branch"


def workload_config(c, world, extra=None, name="c4", per_rank=None):
    if name == "stack":
        d = {
            "workload": "stack: config 5, DEFCON interval-3 DCNv2 stack of R101 C3-C5 (11 layers: "
                        + ", ".join(f"{l.name} {l.H}x{l.W}x{l.Cin}->{l.Ho}x{l.Wo}x{l.Cout} s{l.stride}"
                                    for l in configs.stack_layers(1))
                        + "), bf16, each layer fed by its lightweight offset branch",
            "global_batch": STACK_GLOBAL_BATCH,
            "per_gpu_batch": per_rank,
            "parallelism": f"dp{world} (global batch 64 split by image, strong scaling, no data-path "
                           "collective)",
        }
        if extra:
            d.update(extra)
        return d
    d = {
        "workload": f"{c.name}: N={c.N}/GPU Cin=Cout={c.Cin} {c.H}x{c.W} K={c.K} stride={c.stride} "
                    f"G={c.G} DCNv2 {c.dtype} + lightweight offset branch (dw3x3+BN+ReLU+1x1)",
        "global_batch": c.N * world,
        "parallelism": f"dp{world} (images sharded, no data-path collective)",
    }
    if extra:
        d.update(extra)
    return d


def load_peaks():
    try:
        with open(PEAKS_PATH) as f:
            p = json.load(f)
        return p, "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


# ------------------------------------------------------------------ clocks sampler
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []
        self.t = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))

    def stop(self):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.t is not None:
            self.t.join(timeout=2)

    def summary(self, t0, t1):
        rows = [l for (t, l) in self.lines if t0 - 0.06 <= t <= t1 + 0.06] or [l for _, l in self.lines]
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            parts = [p.strip() for p in r.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


# ------------------------------------------------------------------ GPU arm
class Layer:
    """Device-resident inputs/outputs of one layer's buffer set (one batch of the workload)."""

    def __init__(self, c, images, dev, branch_dev, weight, bias, fp32_mode):
        import paper_conf_ipps_jayaweeralwrk24_b200 as d
        dt = torch.bfloat16 if c.dtype == "bf16" else torch.float32
        self.c = c
        self.fp32_mode = fp32_mode
        self.x = torch.from_numpy(inputs.gen_x(c, images)).to(dev, dt)
        KK = c.K * c.K
        self.off = torch.empty((c.N, c.Ho, c.Wo, c.G, KK, 2), device=dev, dtype=torch.float32)
        self.msk = torch.empty((c.N, c.Ho, c.Wo, c.G, KK), device=dev, dtype=torch.float32)
        self.y = torch.empty((c.N, c.Ho, c.Wo, c.Cout), device=dev, dtype=dt)
        self.branch = branch_dev
        self.weight = weight
        self.bias = bias
        nws = d.defcon_dcn_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout, c.K, c.K, c.stride, c.pad,
                                          c.dil, c.G, dt, fp32_mode=fp32_mode)
        self.ws = torch.zeros(max(nws, 16), dtype=torch.uint8, device=dev)   # zero before first use
        self.tws = torch.empty(d.defcon_offset_workspace_size(c.N, c.H, c.W, c.Cin, c.K, c.stride,
                                                              c.pad, c.dil, c.G),
                               dtype=torch.uint8, device=dev)
        # step 1's parameters packed once, as at model load (defcon_offset_pack_params); layers
        # whose shape runs the two-launch branch keep the per-call path (set in gpu_arm)
        B = branch_dev
        self.packed = d.defcon_offset_pack_params(B["dw_w"], B["dw_scale"], B["dw_shift"], B["pw_w"],
                                                  K=c.K, offset_groups=c.G, with_mask=c.modulated)

    def nbytes(self):
        return sum(t.numel() * t.element_size() for t in (self.x, self.off, self.msk, self.y,
                                                           self.weight))


def step1(d, L):
    c, B = L.c, L.branch
    if L.packed is not None:
        d.defcon_offset_dw_conv_packed(L.x, L.packed, B["pw_b"], K=c.K, stride=c.stride, pad=c.pad,
                                       dil=c.dil, offset_groups=c.G, with_mask=c.modulated,
                                       offset=L.off, mask=L.msk)
        return
    d.defcon_offset_dw_conv(L.x, B["dw_w"], B["dw_scale"], B["dw_shift"], B["pw_w"], B["pw_b"],
                            K=c.K, stride=c.stride, pad=c.pad, dil=c.dil, offset_groups=c.G,
                            with_mask=c.modulated, offset=L.off, mask=L.msk, workspace=L.tws)


def step2(d, L):
    c = L.c
    d.defcon_dcn_forward(L.x, L.off, L.msk, L.weight, L.bias, stride=c.stride, pad=c.pad,
                         dil=c.dil, offset_groups=c.G, y=L.y, workspace=L.ws, fp32_mode=L.fp32_mode)


def capture(fn, stream):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        fn()
    return g


def launches_per_layer(c, fp32_mode, packed=False):
    """Kernels one layer launches: the offset branch (the one-pass kernel from pre-packed
    parameters: 1; else weight-pack + one-pass kernel, or the two-pass dw + 1x1 kernels: 2) + the
    DCN kernel (+ the W tf32 split for 3xTF32)."""
    return (1 if packed else 2) + 1 + (1 if c.dtype == "f32" and fp32_mode == "3xtf32" else 0)


def gpu_arm(args, rank, world, local_rank, dist):
    import paper_conf_ipps_jayaweeralwrk24_b200 as d

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    d.load_library()
    base_layers, fp32_mode, strong = WORKLOADS[args.workload]
    if strong:   # config 5: global batch 64 split over the ranks
        images = sharding.shard_strong(rank, world, STACK_GLOBAL_BATCH)
    else:        # weak scaling: each rank regenerates exactly its own shard of N images
        images = sharding.shard_images(rank, world, base_layers[0].N)
    layers = [l.replace(N=len(images)) for l in base_layers]
    c0 = layers[0]

    def make_set():
        out = []
        for c in layers:
            dt = torch.bfloat16 if c.dtype == "bf16" else torch.float32
            P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
            w, b = inputs.gen_weight(c)
            out.append(Layer(c, images, dev, P, torch.from_numpy(w).to(dev, dt), torch.from_numpy(b).to(dev),
                             fp32_mode))
        return out

    # Rotate buffer sets so the sets touched between two visits exceed L2 (cold-L2 timing).
    sets = [make_set()]
    set_bytes = sum(L.nbytes() for L in sets[0])
    R = max(2, int(np.ceil(1.5 * L2_BYTES / set_bytes))) if set_bytes < 1.5 * L2_BYTES else 1
    sets += [make_set() for _ in range(R - 1)]
    rot_bytes = set_bytes * R

    stream = torch.cuda.Stream(device=dev)
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        for S in sets:          # eager warm-up outside capture (module load, attributes)
            for L in S:
                try:
                    step1(d, L)
                except d.DefconError as e:   # UNSUPPORTED: this shape runs the two-launch branch
                    if e.status != 2:
                        raise
                    L.packed = None
                    step1(d, L)
                step2(d, L)
    torch.cuda.synchronize()

    def whole(S):
        for L in S:
            step1(d, L)
            step2(d, L)

    g_step = [capture(lambda S=S: whole(S), stream) for S in sets]
    g_dcn = [capture(lambda S=S: [step2(d, L) for L in S], stream) for S in sets]
    g_br = [capture(lambda S=S: [step1(d, L) for L in S], stream) for S in sets]
    torch.cuda.synchronize()

    def run(graphs, n):
        for i in range(n):
            graphs[i % R].replay()

    def barrier():
        if dist is not None:
            dist.barrier()

    clk = ClockSampler(local_rank)
    clk.start()
    time.sleep(0.3)
    with torch.cuda.stream(stream):
        run(g_step, args.warmup)
    torch.cuda.synchronize()

    # ---------------- timed region: exactly K steps
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t_wall0 = time.time()
    with torch.cuda.stream(stream):
        e0.record(stream)
        run(g_step, args.steps)
        e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    t_wall1 = time.time()
    ms_total = e0.elapsed_time(e1)
    # keep the GPU busy for clock sampling when the timed region was very short
    if t_wall1 - t_wall0 < 0.5:
        t_ext = time.time()
        with torch.cuda.stream(stream):
            while time.time() - t_ext < 0.6:
                run(g_step, 20)
                torch.cuda.synchronize()
        t_wall1 = time.time()

    # ---------------- per-kernel timing (same rotation), for the roofline
    def time_graphs(graphs, n):
        a, bq = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            run(graphs, 3 * R)
            a.record(stream)
            run(graphs, n)
            bq.record(stream)
        torch.cuda.synchronize()
        return a.elapsed_time(bq) / n

    n_k = max(args.steps, 200 // len(layers))
    ms_dcn = time_graphs(g_dcn, n_k)
    ms_branch = time_graphs(g_br, n_k)
    clk.stop()
    clocks = clk.summary(t_wall0, t_wall1)

    # ---------------- end to end through the C ABI with pinned host buffers: every layer's x
    # from pinned host memory, its y back (defcon_layer_forward_host, one call per layer)
    e2e_in = []
    for L in sets[0]:
        c = L.c
        dt = L.x.dtype
        ws = torch.empty(d.defcon_layer_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout, K=c.K,
                                                       stride=c.stride, pad=c.pad, dil=c.dil,
                                                       offset_groups=c.G, dtype=dt,
                                                       modulated=c.modulated, fp32_mode=fp32_mode),
                         dtype=torch.uint8, device=dev)
        e2e_in.append((L, L.x.cpu().pin_memory(), torch.empty(tuple(L.y.shape), dtype=dt).pin_memory(), ws))

    def e2e_step():
        for L, xh, yh, ws in e2e_in:
            c = L.c
            d.defcon_layer_forward_host(xh, L.branch, L.weight, L.bias, yh, ws, K=c.K,
                                        stride=c.stride, pad=c.pad, dil=c.dil, offset_groups=c.G,
                                        modulated=c.modulated, fp32_mode=fp32_mode, stream=stream)

    e2e_steps = max(3, min(args.steps, 50 // len(layers)))
    with torch.cuda.stream(stream):
        for _ in range(2):
            e2e_step()
        barrier()
        a, bq = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(e2e_steps):
            e2e_step()
        bq.record(stream)
    torch.cuda.synchronize()
    ms_e2e = a.elapsed_time(bq) / e2e_steps
    h2d = sum(xh.numel() * xh.element_size() for _, xh, _, _ in e2e_in)
    d2h = sum(yh.numel() * yh.element_size() for _, _, yh, _ in e2e_in)
    del e2e_in

    # ---------------- collectives outside the timed region: per-image fp64
    # checksums of the last layer's y all-gathered (invariance: an image's y does not depend on
    # its rank), and every rank's y gathered into rank 0, timed on its own
    with torch.cuda.stream(stream):
        y0 = sets[0][-1].y
        cks = sharding.gather_checksums(dist, sharding.image_checksums(y0))
        barrier()
        ga, gb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ga.record(stream)
        yall = sharding.gather_outputs(dist, y0)
        gb.record(stream)
    torch.cuda.synchronize()
    ms_gather = ga.elapsed_time(gb)
    gather_bytes = int(yall.numel() * yall.element_size())
    del yall

    # ---------------- max over ranks
    ms_total, ms_e2e, ms_dcn, ms_branch, ms_gather = sharding.max_over_ranks(
        dist, [ms_total, ms_e2e, ms_dcn, ms_branch, ms_gather], dev)

    flops = sum(configs.contraction_flops(c) for c in layers)       # per rank, per step
    ms_step = ms_total / args.steps
    value = world * flops * args.steps / (ms_total * 1e-3) / 1e12
    peaks, peak_src = load_peaks()
    achieved = flops / (ms_dcn * 1e-3) / 1e12
    f32 = c0.dtype == "f32"
    if f32 and fp32_mode == "3xtf32":   # 3 tf32 MMAs per product; tf32 peak = bf16 peak / 2 (nominal ratio)
        peak, peak_unit_note = peaks["bf16_tflops"] / 2 / 3, "bf16 burst / 2 (tf32) / 3 (3xTF32 products)"
    elif f32:                           # FFMA: 148 SMs x 128 lanes x 2 flop x max SM clock
        peak, peak_unit_note = 148 * 128 * 2 * 1.965e9 / 1e12, "fp32 FFMA (148 x 128 x 2 x 1965 MHz)"
    else:
        peak, peak_unit_note = peaks["bf16_tflops"], "bf16 burst"
    traffic = None
    if args.workload == "c4":
        try:   # dram read+write bytes per launch of the DCN kernel, latest committed ncu capture
            import glob
            latest = sorted(glob.glob(NCU_SUMMARY_GLOB))[-1]
            with open(latest) as f:
                js = json.load(f)
            traffic = js.get("dcn_dram_bytes_per_launch")
            traffic_note = js.get("dcn_dram_bytes_note")
        except Exception:
            traffic_note = None
    kernel = ("dcn_fwd_bf16_tc_kernel<F32> (fused gather + tcgen05 kind::tf32 3xTF32 implicit GEMM)"
              if f32 and fp32_mode == "3xtf32" else
              "dcn_fwd_f32 CUDA-core kernel (FFMA)" if f32 else
              "dcn_fwd_bf16_tc_kernel (fused gather + tcgen05 implicit GEMM)")
    if len(layers) > 1:
        kernel += f", summed over the {len(layers)} layers of the stack"
    per_layer = {}
    if len(layers) > 1:
        per_layer = {"layers": [c.name for c in layers]}
    line = {
        "metric": metric_name(args.workload),
        "value": round(value, 3),
        "unit": "TFLOP/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(ms_step, 5),
        "higher_is_better": True,
        "scaling": "strong" if strong else "weak",
        "vs_baseline": None,
        "dtype": "f32" if f32 else "bf16",
        "data": "synthetic (seeded; x=ReLU(N(0,1)), offsets from the dw offset branch, "
                "random-init weights)",
        "config": workload_config(c0, world, dict({
            "l2": (f"rotating {R} buffer sets ({rot_bytes / 2**20:.0f} MiB > 126 MiB L2), CUDA graphs"
                   if R > 1 else f"inputs larger than L2 ({set_bytes / 2**20:.0f} MiB per step), CUDA graphs"),
            "us_per_step": round(ms_step * 1e3, 2),
            "us_dcn_kernels": round(ms_dcn * 1e3, 2),
            "us_offset_branch_kernels": round(ms_branch * 1e3, 2),
            "fp32_mode": fp32_mode if f32 else None,
            "branch_params": ("packed once outside the timed region (defcon_offset_pack_params, as at model load)"
                              if all(L.packed is not None for L in sets[0]) else "packed per call"),
        }, **per_layer), name=args.workload, per_rank=len(images)),
        "roofline": {
            "kernel": kernel,
            "bound": "tensor" if not (f32 and fp32_mode == "simt") else "alu",
            "achieved": round(achieved, 2),
            "peak": round(peak, 1),
            "peak_source": (f"{peak_src} {peak_unit_note} (MEASURED_PEAKS.json)" if peak_src == "measured"
                            else f"fallback {peak_unit_note} (B200_PROFILING.md)"),
            "unit": "TFLOP/s",
            "frac": round(achieved / peak, 4),
            "traffic": traffic,
        },
        "clocks": clocks,
        "e2e": {
            "value": round(world * flops / (ms_e2e * 1e-3) / 1e12, 3),
            "unit": "TFLOP/s",
            "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h),
            "ms_per_step": round(ms_e2e, 4),
            "api": "defcon_layer_forward_host (C ABI, pinned host x -> y)"
                   + (", one call per layer" if len(layers) > 1 else ""),
        },
        "gpu_launches": args.steps * sum(launches_per_layer(L.c, fp32_mode, L.packed is not None)
                                         for L in sets[0]),
        "collectives": {                  # outside the timed region
            "checksum_images": int(cks.shape[0]),
            "y_checksum_image0": [round(float(v), 6) for v in cks[0].tolist()],
            "y_gather_ms": round(ms_gather, 4),
            "y_gather_bytes": gather_bytes,
        },
    }
    if traffic is not None:
        line["roofline"]["traffic_note"] = traffic_note
    if not f32:   # context: the measured sustained bf16 figure (cuBLAS back to back for 4 s)
        line["roofline"]["peak_sustained"] = peaks.get("bf16_tflops_sustained")
        line["roofline"]["frac_sustained"] = (round(achieved / peaks["bf16_tflops_sustained"], 4)
                                              if peaks.get("bf16_tflops_sustained") else None)
    return line


# ------------------------------------------------------------------ oracle (CPU) legs
def oracle_sample(layers, target_s, images=4):
    """Time the oracle as it stands on a bounded sample of the workload: for every layer, the
    offset branch of `images` images plus the DCN at n_pix of their output pixels (n_pix
    calibrated so the sample takes about target_s seconds); returns (TFLOP/s, seconds,
    description, n_pix, step function)."""
    import oracle
    oracle.build()
    prep = []
    for c in layers:
        ci = c.replace(N=images)
        x = inputs.gen_x(ci, images=list(range(images)))
        P = inputs.gen_offset_branch(c)
        w, b = inputs.gen_weight(c)
        prep.append((c, ci, x, P, w, b))

    def step(n_pix):
        for c, ci, x, P, w, b in prep:
            off, msk = oracle.offset_branch(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"],
                                            P["pw_b"], K=c.K, G=c.G, with_mask=c.modulated,
                                            stride=c.stride, pad=c.pad, dil=c.dil)
            idx = np.arange(n_pix) % ci.M
            oracle.dcn_pixels(x, off, w, idx, b, mask=msk, stride=c.stride, pad=c.pad, dil=c.dil, G=c.G)

    def once(n_pix):
        t0 = time.perf_counter()
        step(n_pix)
        return time.perf_counter() - t0

    t_small = once(256)
    t_big = once(2048)
    per_pix = max((t_big - t_small) / (2048 - 256), 1e-7)
    fixed = max(t_small - 256 * per_pix, 0.0)
    n_pix = int(np.clip((target_s - fixed) / per_pix, 256, 50 * min(l.replace(N=images).M for l in layers)))
    dt = once(n_pix)
    flops = sum(2 * n_pix * c.Cout * c.K * c.K * c.Cin for c in layers)
    what = layers[0].name if len(layers) == 1 else f"each of the {len(layers)} stack layers"
    sample = (f"{what}: offset branch of {images} image(s) + DCN at {n_pix} of their output "
              f"pixels ({flops / 1e9:.1f} GFLOP contraction), fp64 C oracle, OpenMP")
    return flops / dt / 1e12, dt, sample, n_pix, step, flops


def sample_images(name):
    return 1 if name == "stack" else 4


def cpu_baseline(name):
    import oracle
    layers = WORKLOADS[name][0]
    v, dt, sample, _, _, _ = oracle_sample(layers, target_s=10.0, images=sample_images(name))
    out = {"value": v, "unit": "TFLOP/s", "cores": oracle.num_threads(), "kind": "oracle",
           "sample": sample, "seconds": round(dt, 2)}
    # the oracle also single-core on config 1 (the tiny DCNv1 fp32 layer)
    t = configs.TINY
    L = inputs.gen_layer(t)
    ncores = oracle.num_threads()
    oracle.set_num_threads(1)
    try:
        t0 = time.perf_counter()
        oracle.dcn_forward(L["x"], L["offset"], L["weight"], L["bias"], mask=L["mask"])
        t1 = time.perf_counter() - t0
    finally:
        oracle.set_num_threads(ncores)
    out["tiny_1core"] = {"config": t.name, "seconds": round(t1, 4),
                         "tflops": round(configs.contraction_flops(t) / t1 / 1e12, 6)}
    return out


def reference_arm(args, world):
    """--impl reference: the fp64 oracle, as it stands, on the host cores (rank 0 only).
    Each step is a bounded sample of the workload (see oracle_sample), sized so that the
    whole --steps/--warmup run finishes within a few minutes."""
    import oracle
    layers, _, strong = WORKLOADS[args.workload]
    per_step_s = float(np.clip(150.0 / max(args.steps + args.warmup, 1), 1.0, 10.0))
    _, _, sample, n_pix, step, flops = oracle_sample(layers, target_s=per_step_s,
                                                     images=sample_images(args.workload))
    for _ in range(args.warmup):
        step(n_pix)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step(n_pix)
    dt = time.perf_counter() - t0
    value = flops * args.steps / dt / 1e12
    sample = "per step: " + sample
    return {
        "impl": "reference",
        "metric": metric_name(args.workload),
        "value": value,
        "unit": "TFLOP/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True,
        "scaling": "strong" if strong else "weak",
        "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic (seeded)",
        "config": workload_config(layers[0], world, {"sample": sample}, name=args.workload,
                                  per_rank=STACK_GLOBAL_BATCH // world if strong else None),
        "cpu_baseline": {"value": value, "unit": "TFLOP/s", "cores": oracle.num_threads(),
                         "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=50)
    ap.add_argument("--impl", default="defcon", choices=["defcon", "reference"])
    ap.add_argument("--workload", default="c4", choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        if rank == 0:
            print(json.dumps(reference_arm(args, world)), flush=True)
        return

    dist = None
    if world > 1:
        import torch.distributed as tdist
        torch.cuda.set_device(local_rank)
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        dist = tdist
    line = gpu_arm(args, rank, world, local_rank, dist)
    if rank == 0:
        if not args.no_cpu_baseline and world == 1:
            line["cpu_baseline"] = cpu_baseline(args.workload)
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
