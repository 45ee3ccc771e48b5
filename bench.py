#!/usr/bin/env python
"""Benchmark: the B200 quantized-conv library on the paper's workloads (BASELINE.json).

Default workload = BASELINE configs[4] ("C5"): the ResNet-50 conv trunk at A4W4, global
batch 256, batch-sharded over the GPUs (strong scaling: 256/G images per GPU; `--batch B`
gives weak scaling with B images per GPU).  One step = the whole hot path (SURVEY.md 8(a)
rows a1, a3-a6) over one batch: the 53 ResNet-50 conv layers chained in network order --
the stem takes the fp32 image (qconv2d_forward_quantize: the quantization to codes runs
inside the stem kernel, space-to-depth form), the other 52 take the previous layer's packed
codes (qconv2d_forward: implicit GEMM on tcgen05 tensor cores with bias / re-quantization /
ReLU / packing fused).  Weight and
parameter preparation (row a2) happens once, off the timed path; with N GPUs rank 0's
weights are broadcast once over NCCL -- the only collective (row e).

After the timed region the GPU result is checked against the CPU oracle: the first and last
image of the rank's shard go through the oracle's chain of all 53 layers and every layer's
output bytes are compared (`parity` key).

Other workloads (`--workload`), one JSON line each, for the per-layer configurations:
  c1  BASELINE configs[0]: 8-bit 3x3 C=K=64 56x56, batch 1 -- latency, L2 flushed per launch
  c2  BASELINE configs[1]: the same layer at A4W4 with the fused fp32 quantize -> conv
  c3  BASELINE configs[2]: every ResNet-50 conv layer at batch 32 (`--bits` 4 or 8)
  c4  BASELINE configs[3]: the VGG-16 conv stack at 8 bits, batch 64
  f4  SURVEY row f4: the paper's 19 unique ResNet-50 layers at batch 1 and 16 (Fig.10) and
      the DenseNet-121 conv shapes (Fig.17) at batch 1
Prints ONE JSON line (rank 0).  `--impl reference` times the CPU oracle (test
infrastructure, oracle/) on a bounded sample instead.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "ResNet-50 conv-layer TOPS (4/8-bit) vs int8 peak; images/s at 1/2/4/8 GPUs"
GLOBAL_BATCH = 256          # BASELINE configs[4]


def load_peaks():
    """Roofline denominators: MEASURED_PEAKS.json (int8 dense = 2 x bf16 dense, the nominal
    4.5 / 2.25 PFLOP/s ratio of B200_PROFILING.md).  The conv launches are 5-250 us kernels
    in a 2-3 ms step at the maximum SM clock with no power cap active (the clocks key of every
    run shows it), so the burst figure is the one that applies; the sustained one is
    reported beside it."""
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return dict(hbm_gbs=float(d["hbm_gbs"]), int8_tops=2.0 * float(d["bf16_tflops"]),
                    int8_tops_sustained=2.0 * float(d.get("bf16_tflops_sustained", d["bf16_tflops"])),
                    source="measured (MEASURED_PEAKS.json; int8 = 2 x bf16 burst)")
    return dict(hbm_gbs=6650.0, int8_tops=2 * 1590.0, int8_tops_sustained=2 * 1400.0,
                source="fallback (B200_PROFILING.md; int8 = 2 x bf16)")


def measured_traffic(bits: int, batch: int):
    """DRAM bytes (read + write) of the 53 conv launches of one step, from the newest ncu
    launch list summarised under profiles/ (only for the configuration it was measured on)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_traffic.json")))
    for fn in reversed(files):
        with open(fn) as f:
            d = json.load(f)
        if d.get("bits", 4) == bits and d.get("batch", 256) == batch:
            return d["conv_dram_bytes_per_step"]
    return None


def layer_algorithmic(cs: W.ConvShape, bits: int):
    """Algorithmic ops (2 x MAC with the true C) and bytes (touched input + weights +
    output + 12 B/channel of params) of one layer launch."""
    ops = 2 * cs.macs
    touched = cs.h * cs.w if (cs.r > 1 or cs.stride == 1) else cs.p * cs.q
    b = bits / 8
    nbytes = cs.n * touched * cs.c * b + cs.k * cs.r * cs.s * cs.c * b + \
        cs.n * cs.p * cs.q * cs.k * b + 12 * cs.k
    return ops, nbytes


def roofline_us(ops, nbytes, peaks):
    """Per-launch roofline time: the slower of the tensor pipe and HBM."""
    return max(ops / (peaks["int8_tops"] * 1e12), nbytes / (peaks["hbm_gbs"] * 1e9)) * 1e6


def shard_bounds(rank: int, world: int, global_batch: int):
    """Contiguous batch slice of rank `rank`: images [start, start+count)."""
    base, extra = divmod(global_batch, world)
    count = base + (1 if rank < extra else 0)
    start = rank * base + min(rank, extra)
    return start, count


def broadcast_params(dist, tensors, src: int = 0):
    """The only collective of the path: rank `src`'s weights/params to every rank, once."""
    for t in tensors:
        dist.broadcast(t, src=src)


# ----------------------------------------------------------------------------- trunk
def trunk_layers(bits: int, batch: int):
    """(ConvShape, stored C, layer index) in network order for the bench trunk."""
    return [(cs, W.stored_channels(cs, bits), i) for i, cs in enumerate(W.resnet50_convs(batch))]


def stem_scale(bits: int) -> float:
    return 3.0 / 15 if bits == 4 else 3.0 / 255


class Trunk:
    """The 53 ResNet-50 conv layers resident on one GPU (C5's per-rank shard)."""

    def __init__(self, bits: int, batch: int, device, dist_ctx=None, rank: int = 0, stem_dtype: str = "bf16"):
        import torch
        import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
        self.qc = qc
        self.bits = bits
        self.batch = batch
        self.device = device
        self.layers = []
        x_t = W.U4 if bits == 4 else W.U8
        w_t = W.S4 if bits == 4 else W.S8
        self.x_t = x_t
        rank0 = dist_ctx is None or dist_ctx["rank"] == 0
        specs = trunk_layers(bits, batch)
        # ---- weights + params: generated on rank 0, broadcast once (the only collective)
        params = []
        for cs, c_st, i in specs:
            stem = i == 0
            if rank0:
                lp = W.make_layer_params(cs, bits, W.layer_seed(i), c_store=None if stem else c_st)
                # stem: C = 3 codes stored one per byte (space-to-depth path)
                wbytes = W.pack_codes(lp.w_codes, W.S8) if stem else lp.w_bytes
                wb = torch.from_numpy(np.ascontiguousarray(wbytes).reshape(-1)).to(device)
                m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
                pb = torch.from_numpy(np.stack([lp.bias, m, n]).astype(np.int32)).to(device)
            else:
                nbytes = cs.k * cs.r * cs.s * (cs.c if stem else c_st * bits // 8)
                wb = torch.empty(nbytes, dtype=torch.uint8, device=device)
                pb = torch.empty((3, cs.k), dtype=torch.int32, device=device)
            if dist_ctx is not None and dist_ctx["world"] > 1:
                broadcast_params(dist_ctx["dist"], (wb, pb))
            params.append((wb, pb))
        # ---- activations (seeded per rank)
        g = torch.Generator(device=device)
        g.manual_seed(W.SEED_BASE + 7919 * rank)
        stem = specs[0][0]
        self.x_float = torch.relu(torch.randn((batch, stem.h, stem.w, stem.c), generator=g,
                                              device=device, dtype=torch.float32))
        # the image as the stem reads it: bf16 (default; half the bytes over PCIe and HBM, the
        # quantize takes the exact fp32 value of each bf16) or fp32
        self.stem_dtype = stem_dtype
        if stem_dtype == "bf16":
            self.x_float = self.x_float.to(torch.bfloat16)
        self.s_in = stem_scale(bits)
        # the stem (7x7/s2, C=3) takes the fp32 image: qconv2d_forward_quantize runs it as one
        # kernel (the fp32 rows are quantized inside it, straight into its space-to-depth
        # operand tile: 4x4/s1 over 16 byte-coded channels)
        self.stem_desc = qc.make_desc(batch, stem.h, stem.w, stem.c, stem.k, stem.r, stem.s,
                                      stride=stem.stride, pad=stem.pad, x_t=x_t, w_t=W.S8,
                                      y_t=x_t, relu=True)
        # res2 input: max-pool is outside the method -> separately drawn codes
        rng = np.random.default_rng(W.SEED_BASE + 31 * rank + 1)
        codes = W.post_relu_codes_fast(rng, (batch, 56, 56, 64), bits)
        if bits == 4:
            packed = (codes[..., 0::2] | (codes[..., 1::2] << 4)).astype(np.uint8)
        else:
            packed = codes
        self.res2_host = packed
        self.res2_in = torch.from_numpy(packed).to(device)
        cur = None
        block_in = None
        for (cs, c_st, i), (wb, pb) in zip(specs, params):
            if i == 0:
                d = qc.qconv_desc.from_buffer_copy(self.stem_desc)
                w_prep = qc.qconv_prepare_weights(d, wb)
                d.w_prepared = 1
            else:
                d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride,
                                 pad=cs.pad, x_t=x_t, w_t=w_t, y_t=x_t, relu=True)
                w_prep = qc.qconv_prepare_weights(d, wb)
                d.w_prepared = 1
            p, q = qc.out_hw(d)
            y = torch.empty((cs.n, p, q, cs.k * bits // 8), dtype=torch.uint8, device=device)
            role = W.RESNET50_LAYERS[i]["role"]
            if role == "stem":
                src = self.x_float
            elif role == "2a":
                block_in = self.res2_in if cs.name.startswith("res2a") else cur
                src = block_in
            elif role == "branch1":
                src = block_in
            else:
                src = cur
            assert src.shape[1] == d.h and src.shape[2] == d.w, cs.name
            ops, nbytes = layer_algorithmic(cs, bits)
            if i == 0:                      # the stem reads the float image, not codes
                nbytes += cs.n * cs.h * cs.w * cs.c * (self.x_float.element_size() - bits / 8)
            plan = qc.qconv_debug_plan_quantize(d) if i == 0 else qc.qconv_debug_plan(d)
            self.layers.append(dict(name=cs.name, shape=cs, desc=d, w=w_prep, bias=pb[0], m=pb[1],
                                    n=pb[2], x=src, y=y, ops=ops, bytes=nbytes, plan=plan))
            if role in ("stem", "2a", "2b", "2c"):
                cur = y
        self.out = cur
        torch.cuda.synchronize()

    @property
    def ops_per_step(self):
        return sum(L["ops"] for L in self.layers)

    def launches_per_step(self):
        return len(self.layers)

    def step(self, events=None, x_float=None, before_last=None):
        """Enqueue one step on the current stream; events[i] recorded after launch i;
        before_last() runs just before the last layer is enqueued (e2e: the wait for the D2H
        of the previous step's output, which that layer overwrites)."""
        qc = self.qc
        last = len(self.layers) - 1
        for j, L in enumerate(self.layers):
            if j == last and before_last is not None:
                before_last()
            if j == 0:                  # fused fp32 quantize + stem
                qc.qconv2d_forward_quantize(L["desc"], self.x_float if x_float is None else x_float,
                                            self.s_in, L["w"], L["bias"], L["m"], L["n"], y=L["y"])
            else:
                qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
            if events is not None:
                events[j].record()


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    def __init__(self, index: int, period_s: float = 0.01):
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:  # pragma: no cover
            self.ok = False
        self.period = period_s

    def _run(self):
        nv = self.nv
        names = {
            "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4,
            "hw_slowdown": 0x8, "sync_boost": 0x10, "sw_thermal_slowdown": 0x20,
            "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80,
            "display_clock_setting": 0x100,
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in names.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(self.period)

    def start(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()

    def stop(self):
        if self._t is not None:
            self._stop.set()
            self._t.join()
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


# ----------------------------------------------------------------------------- oracle legs
class OracleTrunk:
    """The CPU oracle (test infrastructure, as it stands) on the same trunk, one image at a
    time: quantize the fp32 stem input, then the 53 layers chained as in Trunk.  Weights and
    scales are regenerated from the same seeds; (m, shift) come from the oracle's R1."""

    def __init__(self, bits: int, stem_dtype: str = "bf16"):
        import oracle
        self.oracle = oracle
        self.bits = bits
        self.bf16 = stem_dtype == "bf16"   # image() draws the stem input as the bench does
        self.cores = os.cpu_count() or 1
        os.environ.setdefault("OMP_NUM_THREADS", str(self.cores))
        self.x_t = W.U4 if bits == 4 else W.U8
        self.specs = [(cs, 4 if i == 0 else c_st, i) for cs, c_st, i in trunk_layers(bits, 1)]
        self.lps = [W.make_layer_params(cs, bits, W.layer_seed(i), c_store=c_st)
                    for cs, c_st, i in self.specs]
        self.mns = [oracle.requant_params(lp.s_x, lp.s_w, lp.s_y) for lp in self.lps]
        self.ops = [2 * cs.macs for cs, _, _ in self.specs]
        self.rng = np.random.default_rng(5)

    def _run_layer(self, j, src):
        cs, c_st, i = self.specs[j]
        lp = self.lps[j]
        m, n = self.mns[j]
        return self.oracle.conv2d(src, lp.w_bytes, n=src.shape[0], h=cs.h, wd=cs.w, c=c_st, k=cs.k,
                                  r=cs.r, s=cs.s, xt=self.x_t, wt=lp.w_t, yt=self.x_t,
                                  stride=(cs.stride, cs.stride), pad=(cs.pad, cs.pad),
                                  clamp_lo=lp.clamp_lo, clamp_hi=lp.clamp_hi, bias=lp.bias,
                                  mult=m, shift=n)

    def chain(self, xf, res2, layer_subset=None, bf16=False):
        """xf: fp32 [1,224,224,3] stem input (bf16=True: its uint16 bf16 bit patterns), res2:
        packed res2 input codes [1,56,56,*].  Returns (outputs per layer -- None where
        skipped --, ops done)."""
        xq = self.oracle.quantize(xf, stem_scale(self.bits), 0, self.x_t, c_pad=self.specs[0][1], bf16=bf16)
        subset = range(len(self.specs)) if layer_subset is None else layer_subset
        cur = block_in = None
        outs, ops = [], 0
        for j, (cs, c_st, i) in enumerate(self.specs):
            role = W.RESNET50_LAYERS[i]["role"]
            if role == "stem":
                src = xq
            elif role == "2a":
                block_in = res2 if cs.name.startswith("res2a") else cur
                src = block_in
            elif role == "branch1":
                src = block_in
            else:
                src = cur
            if j in subset:
                y = self._run_layer(j, src)
                ops += self.ops[j]
            else:
                # outside the sampled subset: a stand-in activation of the right shape
                y = np.zeros((xf.shape[0], cs.p, cs.q, cs.k * self.bits // 8), dtype=np.uint8)
            outs.append(y if j in subset else None)
            if role in ("stem", "2a", "2b", "2c"):
                cur = y
        return outs, ops

    def image(self, layer_subset=None):
        """One random image through quantize + (a subset of) the layers; returns ops done."""
        xf = np.maximum(self.rng.standard_normal((1, 224, 224, 3), dtype=np.float32), 0)
        if self.bf16:      # round to nearest even bf16 bit patterns (finite inputs)
            u = xf.view(np.uint32).astype(np.uint64)
            xf = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16).astype(np.uint16)
        codes = W.post_relu_codes_fast(self.rng, (1, 56, 56, 64), self.bits)
        res2 = (codes[..., 0::2] | (codes[..., 1::2] << 4)).astype(np.uint8) if self.bits == 4 else codes
        return self.chain(xf, res2, layer_subset, bf16=self.bf16)[1]

    def groups(self, n_groups: int):
        tot = sum(self.ops)
        out, cur, acc = [], [], 0
        for j in range(len(self.specs)):
            cur.append(j)
            acc += self.ops[j]
            if acc >= tot / n_groups and len(out) < n_groups - 1:
                out.append(cur)
                cur, acc = [], 0
        if cur:
            out.append(cur)
        return out


def verify_trunk(trunk: Trunk, images, ot: OracleTrunk = None):
    """Bench self-check (after the timed region): the rank's images `images` through the
    oracle chain; every layer's GPU output bytes of those images must equal the oracle's."""
    import torch
    if ot is None:
        ot = OracleTrunk(trunk.bits)
    t0 = time.perf_counter()
    bad = []
    for img in images:
        xt = trunk.x_float[img:img + 1].cpu()
        bf16 = xt.dtype == torch.bfloat16
        xf = xt.view(torch.int16).numpy().view(np.uint16) if bf16 else xt.numpy()
        outs, _ = ot.chain(xf, trunk.res2_host[img:img + 1], bf16=bf16)
        for L, ref in zip(trunk.layers, outs):
            got = L["y"][img:img + 1].cpu().numpy()
            if not np.array_equal(got, ref):
                bad.append({"image": int(img), "layer": L["name"],
                            "mismatches": int((got != ref).sum())})
    return {"images": [int(i) for i in images], "layers": len(trunk.layers),
            "bit_exact": not bad, "mismatch": bad[:5], "oracle_s": time.perf_counter() - t0}


def oracle_trunk_images_per_s(bits: int, budget_s: float = 15.0, max_images: int = 8, stem_dtype: str = "bf16"):
    """cpu_baseline leg: whole images through the oracle trunk within a time budget."""
    ot = OracleTrunk(bits, stem_dtype)
    ops_img = sum(ot.ops)
    done_ops = 0
    t0 = time.perf_counter()
    n = 0
    while n < max_images and (n == 0 or time.perf_counter() - t0 < budget_s):
        done_ops += ot.image()
        n += 1
    dt = time.perf_counter() - t0
    return done_ops / ops_img / dt, ot.cores, n, dt


def run_reference(args):
    """--impl reference: the oracle, as it stands, on the host cores.  Each step is a
    bounded sample: one image through one of 8 groups of consecutive layers (about 1/8
    of the trunk's ops, rotating); images/s = (ops done / ops per image) / time."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    ot = OracleTrunk(args.bits, args.stem_dtype)
    groups = ot.groups(8)
    ops_img = sum(ot.ops)
    for s in range(args.warmup):
        ot.image(set(groups[s % len(groups)]))
    t = 0.0
    done = 0
    for s in range(args.steps):
        g = set(groups[s % len(groups)])
        t0 = time.perf_counter()
        done += ot.image(g)
        t += time.perf_counter() - t0
    value = done / ops_img / t
    gb = args.global_batch
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "images/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1000 * t / max(args.steps, 1), "higher_is_better": True,
        "scaling": "weak" if args.batch else "strong", "vs_baseline": None, "dtype": "int64",
        "data": "synthetic",
        "config": {"workload": f"resnet50_conv_trunk_a{args.bits}w{args.bits}",
                   "global_batch": gb if not args.batch else args.batch * args.gpus},
        "cpu_baseline": {"value": value, "unit": "images/s", "cores": ot.cores, "kind": "oracle",
                         "sample": "per step: 1 image through 1 of 8 rotating layer groups "
                                   "(+ the stem quantize), ops-weighted"},
        "e2e": {"value": value, "unit": "images/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------- trunk run
def run_trunk(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local_rank)
    device = torch.device("cuda", local_rank)
    dist_ctx = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=device)
        dist_ctx = dict(dist=dist, rank=rank, world=world)
    if args.batch:                                     # weak scaling: B images per GPU
        per_gpu, global_batch, scaling = args.batch, args.batch * world, "weak"
    else:                                              # C5: 256 images over all GPUs
        per_gpu = shard_bounds(rank, world, args.global_batch)[1]
        global_batch, scaling = args.global_batch, "strong"
    from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning
    plans_path = args.plans if args.plans not in ("", "none") else None
    if args.plans == "":
        auto = os.path.join(ROOT, "plans", f"resnet50_trunk_a{args.bits}_b{per_gpu}.json")
        plans_path = auto if os.path.exists(auto) else None
    n_plans = tuning.load_plans(plans_path) if plans_path else 0
    trunk = Trunk(args.bits, per_gpu, device, dist_ctx, rank=rank, stem_dtype=args.stem_dtype)
    plans_note = (f"profile-run table {os.path.relpath(plans_path, ROOT)} ({n_plans} shapes)"
                  if n_plans else "default rule")
    if args.tune:
        entries = tuning.tune_layers(trunk.layers[1:], iters=5)     # the stem runs in s2d form
        for L in trunk.layers[1:]:
            L["plan"] = trunk.qc.qconv_debug_plan(L["desc"])
        plans_note = "autotuned in this run"
        if args.save_plans and rank == 0:
            os.makedirs(os.path.dirname(os.path.abspath(args.save_plans)), exist_ok=True)
            tuning.save_plans(args.save_plans, entries,
                              {"workload": f"resnet50_trunk_a{args.bits}", "per_gpu_batch": per_gpu,
                               "how": "qconv_autotune, 5 timed launches per candidate, CUDA events"})

    if args.profile_steps:
        for _ in range(args.warmup + args.profile_steps):
            trunk.step()
        torch.cuda.synchronize()
        return 0

    stream = torch.cuda.Stream(device=device)
    nL = trunk.launches_per_step()
    # (1) the timed region: one CUDA graph of the whole step with nothing inside but the
    #     53 launches (the conv kernels use programmatic dependent launch, so a kernel's
    #     prologue overlaps the previous kernel's tail -- timing events between launches
    #     would serialize that), replayed K times
    # (2) a second pass, right after, of K graphs with a timing event after every launch:
    #     the per-launch device durations behind the roofline numbers
    graphs, evsets = [], []
    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            trunk.step()
        torch.cuda.synchronize()
        g_plain = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_plain, stream=stream):
            trunk.step()
        for _ in range(args.steps):
            ev = [torch.cuda.Event(enable_timing=True, external=True) for _ in range(nL)]
            start = torch.cuda.Event(enable_timing=True, external=True)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                start.record()
                trunk.step(events=ev)
            graphs.append(g)
            evsets.append([start] + ev)
        for _ in range(max(3, args.warmup)):
            g_plain.replay()
        for g in graphs[: max(3, args.warmup)]:
            g.replay()
    torch.cuda.synchronize()

    clk = ClockSampler(local_rank)
    if dist_ctx:
        dist_ctx["dist"].barrier()
    torch.cuda.synchronize()
    clk.start()
    t_begin = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        t_begin.record()
        for _ in range(args.steps):
            g_plain.replay()
        t_end.record()
    torch.cuda.synchronize()
    if dist_ctx:
        dist_ctx["dist"].barrier()
    torch.cuda.synchronize()
    clocks = clk.stop()
    elapsed_ms = t_begin.elapsed_time(t_end)
    # instrumented pass: per-launch device durations
    i_begin = torch.cuda.Event(enable_timing=True)
    i_end = torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        i_begin.record()
        for g in graphs:
            g.replay()
        i_end.record()
    torch.cuda.synchronize()
    instr_ms_per_step = i_begin.elapsed_time(i_end) / args.steps
    per_launch = np.zeros((args.steps, nL))
    for s, evs in enumerate(evsets):
        for j in range(nL):
            per_launch[s, j] = evs[j].elapsed_time(evs[j + 1])
    if dist_ctx:
        t = torch.tensor([elapsed_ms], device=device, dtype=torch.float64)
        dist_ctx["dist"].all_reduce(t, op=dist_ctx["dist"].ReduceOp.MAX)
        elapsed_ms = float(t.item())
    ms_per_step = elapsed_ms / args.steps
    value = global_batch / (ms_per_step / 1000.0)

    peaks = load_peaks()
    conv_ms = per_launch.mean(axis=0)                  # per conv layer, averaged over steps
    conv_ops = np.array([L["ops"] for L in trunk.layers], dtype=np.float64)
    conv_bytes = np.array([L["bytes"] for L in trunk.layers], dtype=np.float64)
    conv_total_ms = float(conv_ms.sum())
    achieved_tops = conv_ops.sum() / (conv_total_ms / 1e3) / 1e12
    ridge = peaks["int8_tops"] * 1e12 / (peaks["hbm_gbs"] * 1e9)
    cb = conv_ops / conv_bytes >= ridge
    cb_tops = float(conv_ops[cb].sum() / (conv_ms[cb].sum() / 1e3) / 1e12) if cb.any() else None
    roof_us = np.array([roofline_us(o, b, peaks) for o, b in zip(conv_ops, conv_bytes)])
    families = {}
    for j, L in enumerate(trunk.layers):
        f = families.setdefault(L["plan"]["kernel_name"], {"launches": 0, "us": 0.0, "roofline_us": 0.0})
        f["launches"] += 1
        f["us"] += conv_ms[j] * 1e3
        f["roofline_us"] += roof_us[j]
    for f in families.values():
        f["frac"] = f["roofline_us"] / f["us"]
    dominant = max(families, key=lambda k: families[k]["us"])

    e2e = None
    if not args.no_e2e:
        e2e = measure_e2e(trunk, stream, args, global_batch, dist_ctx, device)

    parity = None
    if not args.no_verify:
        parity = verify_trunk(trunk, sorted({0, per_gpu - 1}))
        if dist_ctx:
            ok = torch.tensor([1 if parity["bit_exact"] else 0], device=device)
            dist_ctx["dist"].all_reduce(ok, op=dist_ctx["dist"].ReduceOp.MIN)
            parity["all_ranks_bit_exact"] = bool(ok.item())

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        ips, cores, n_img, dt = oracle_trunk_images_per_s(args.bits, stem_dtype=args.stem_dtype)
        cpu = {"value": ips, "unit": "images/s", "cores": cores, "kind": "oracle",
               "sample": f"{n_img} image(s) x (quantize + 53 layers), {dt:.1f} s"}

    if rank == 0:
        layers = []
        for j, L in enumerate(trunk.layers):
            t_s = conv_ms[j] / 1e3
            layers.append({"name": L["name"], "us": conv_ms[j] * 1e3, "kernel": L["plan"]["kernel_name"],
                           "bn": L["plan"]["bn"], "tops": L["ops"] / t_s / 1e12,
                           "gbs": L["bytes"] / t_s / 1e9, "roofline_us": roof_us[j],
                           "frac_roofline": roof_us[j] / (conv_ms[j] * 1e3),
                           "frac_tensor": L["ops"] / t_s / 1e12 / peaks["int8_tops"],
                           "frac_hbm": L["bytes"] / t_s / 1e9 / peaks["hbm_gbs"]})
        if args.layers_json:
            with open(args.layers_json, "w") as f:
                json.dump({"layers": layers, "families": families,
                           "ms_per_step": ms_per_step}, f, indent=1)
        line = {
            "metric": METRIC, "value": value, "unit": "images/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": f"int{args.bits} (int8 tcgen05 MMA, int32 acc)",
            "data": "synthetic (seeded; random-init weights of ResNet-50 conv shapes)",
            "config": {"workload": f"resnet50_conv_trunk_a{args.bits}w{args.bits}",
                       "global_batch": global_batch, "per_gpu_batch": per_gpu,
                       "layers": len(trunk.layers), "parallelism": f"dp{world} (batch shards)",
                       "stem_input": f"{trunk.stem_dtype} NHWC image, quantized inside the stem kernel",
                       "l2": f"working set > L2: ~2.4 GB of trunk traffic per step (at 256 images per GPU) "
                             f"streams through the 126 MB L2, evicting the {trunk.x_float.numel() * trunk.x_float.element_size() / 1e6:.0f} MB "
                             f"{trunk.stem_dtype} stem input before the next step reads it",
                       "graph": "one CUDA graph per step (PDL between the conv kernels), replayed",
                       "plans": plans_note},
            "tops": trunk.ops_per_step / (ms_per_step / 1e3) / 1e12,
            "roofline": {"bound": "tensor", "kernel": "the 53 conv launches (qconv_halo / qconv_t / qconv_fwd / qconv_fwd2 kernels)",
                         "achieved": achieved_tops, "peak": peaks["int8_tops"],
                         "unit": "TOPS", "frac": achieved_tops / peaks["int8_tops"],
                         "traffic": measured_traffic(args.bits, per_gpu),
                         "traffic_unit": "DRAM bytes per step over the 53 conv launches (ncu, profiles/)",
                         "peak_source": peaks["source"],
                         "peak_sustained": peaks["int8_tops_sustained"],
                         "frac_of_roofline_time": float(roof_us.sum() / (conv_total_ms * 1e3)),
                         "roofline_time_note": "sum over launches of max(ops / int8 peak, bytes / HBM peak) "
                                               "divided by the summed measured launch times",
                         "families": families, "dominant_family": dominant,
                         "conv_share_of_step": conv_total_ms / instr_ms_per_step,
                         "compute_bound_layers": {"count": int(cb.sum()), "ridge_ops_per_byte": ridge,
                                                  "achieved": cb_tops,
                                                  "frac": None if cb_tops is None else cb_tops / peaks["int8_tops"]},
                         "launch_times": "CUDA events after every launch, second pass of K instrumented "
                                         "graph replays right after the timed region",
                         "instrumented_ms_per_step": instr_ms_per_step,
                         "algorithmic_ops_per_step": float(conv_ops.sum()),
                         "algorithmic_bytes_per_step": float(conv_bytes.sum())},
            "quantize_pack": {"kernel": "fused into the stem (qconv2d_forward_quantize: the halo kernel's "
                                        "converter warps quantize the TMA-loaded fp32 rows)",
                              "stem_us": conv_ms[0] * 1e3,
                              "stem_algorithmic_bytes": float(conv_bytes[0])},
            "parity": parity,
            "e2e": e2e, "cpu_baseline": cpu, "clocks": clocks,
            "gpu_launches": args.steps * nL,   # our kernels in the timed region
        }
        print(json.dumps(line), flush=True)
    if dist_ctx:
        dist_ctx["dist"].barrier()
        dist_ctx["dist"].destroy_process_group()
    return 0


def measure_e2e(trunk, stream, args, global_batch, dist_ctx, device):
    """Same metric through the public API with HOST buffers: per step, H2D of the fp32
    stem input from pinned memory, the whole trunk, D2H of the final activation.  The copies
    run on their own streams, double-buffered: step i+1's input crosses PCIe while step i
    computes, and only the last layer of step i waits for the D2H of step i-1's output (the
    buffer that layer overwrites)."""
    import torch
    xh = trunk.x_float.cpu().pin_memory()
    out = trunk.out
    yh = torch.empty(out.shape, dtype=out.dtype, pin_memory=True)
    xd = [torch.empty_like(trunk.x_float) for _ in range(2)]
    steps = max(3, min(args.steps, 20))
    h2d = torch.cuda.Stream(device=device)
    d2h = torch.cuda.Stream(device=device)

    def run(n):
        copied = [None, None]       # H2D done, per input buffer
        consumed = [None, None]     # the step that read the buffer is done
        read_out = [None]           # the D2H of the previous step's output is done
        for i in range(n):
            k = i % 2
            with torch.cuda.stream(h2d):
                if consumed[k] is not None:
                    h2d.wait_event(consumed[k])
                xd[k].copy_(xh, non_blocking=True)
                copied[k] = torch.cuda.Event()
                copied[k].record(h2d)
            with torch.cuda.stream(stream):
                stream.wait_event(copied[k])
                prev = read_out[0]
                trunk.step(x_float=xd[k],
                           before_last=(lambda: stream.wait_event(prev)) if prev is not None else None)
                consumed[k] = torch.cuda.Event()
                consumed[k].record(stream)
            with torch.cuda.stream(d2h):
                d2h.wait_event(consumed[k])
                yh.copy_(out, non_blocking=True)
                read_out[0] = torch.cuda.Event()
                read_out[0].record(d2h)
        return read_out[0]

    run(2)
    torch.cuda.synchronize()
    if dist_ctx:
        dist_ctx["dist"].barrier()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record(stream)
    h2d.wait_stream(stream)          # the first copy starts inside the timed region
    last = run(steps)
    stream.wait_event(last)
    b.record(stream)
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    if dist_ctx:
        t = torch.tensor([ms], device=device, dtype=torch.float64)
        dist_ctx["dist"].all_reduce(t, op=dist_ctx["dist"].ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / steps
    return {"value": global_batch / (ms_step / 1e3), "unit": "images/s",
            "h2d_bytes_per_step": int(xh.numel() * xh.element_size()),
            "d2h_bytes_per_step": int(yh.numel() * yh.element_size()),
            "ms_per_step": ms_step, "steps": steps,
            "note": "public-API launches (eager); H2D of step i+1 and D2H of step i-1 overlap step i "
                    "on separate streams (double-buffered input; only the last layer waits for the "
                    "previous D2H)"}


# ----------------------------------------------------------------------------- per-layer workloads
def workload_layers(name: str, bits: int):
    """(ConvShape list, bits) of the per-layer workloads."""
    if name in ("c1", "c2"):
        return [W.C1]
    if name == "c3":
        return W.resnet50_convs(32)
    if name == "c4":
        return W.vgg16_convs(64)
    if name == "f4":
        return ([cs.with_batch(1) for cs in W.resnet50_unique(1)] +
                [cs.with_batch(16) for cs in W.resnet50_unique(1)] +
                W.densenet121_unique(1))
    raise ValueError(name)


def run_layers(args):
    """Per-layer workloads (C1-C4, f4): each layer launched K times after W warm-ups, L2
    flushed (a 512 MB write) before every timed launch, CUDA events around the launch (and,
    for c2, the fused fp32 quantize before it).  One JSON line for the whole workload."""
    import torch
    import oracle
    import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    device = torch.device("cuda", 0)
    torch.cuda.set_device(device)
    bits = 8 if args.workload in ("c1", "c4") else (4 if args.workload == "c2" else args.bits)
    peaks = load_peaks()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=device)
    shapes = workload_layers(args.workload, bits)
    results, bad, tuned = [], [], []
    total_ops = total_us = total_roof = 0.0
    clk = ClockSampler(0)
    clk.start()
    for i, cs in enumerate(shapes):
        c_st = cs.c if bits == 8 else cs.c + (cs.c % 2)           # 4-bit rows: even channel count
        x_t, w_t = (W.U4, W.S4) if bits == 4 else (W.U8, W.S8)
        lp = W.make_layer_params(cs, bits, W.layer_seed(100 + i), c_store=c_st)
        d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad,
                         x_t=x_t, w_t=w_t, y_t=x_t, relu=True)
        m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
        w = qc.qconv_prepare_weights(d, torch.from_numpy(np.ascontiguousarray(lp.w_bytes)).to(device))
        d.w_prepared = 1
        b = torch.from_numpy(lp.bias).to(device)
        mm, nn = torch.from_numpy(m).to(device), torch.from_numpy(n).to(device)
        xf = None
        if args.workload == "c2":
            g = torch.Generator(device=device)
            g.manual_seed(W.SEED_BASE)
            xf = torch.relu(torch.randn((cs.n, cs.h, cs.w, cs.c), generator=g, device=device))
            x = qc.qconv_quantize_pack(xf, 3.0 / 15, 0, x_t)
        else:
            x = W.device_post_relu_codes((cs.n, cs.h, cs.w, c_st), bits, W.layer_seed(200 + i), device)
        y = qc.qconv2d_forward(d, x, w, b, mm, nn)
        if args.tune:
            best, tus = qc.qconv_autotune(d, x, w, b, mm, nn, y=y, iters=5)
            from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning
            tuned.append({"name": cs.name, "desc": tuning.desc_fields(d), "kernel": best["kernel"],
                          "kernel_name": best["kernel_name"], "bn": best["bn"], "us": tus})
        plan = qc.qconv_debug_plan(d)

        def launch():
            if xf is not None:
                qc.qconv_quantize_pack(xf, 3.0 / 15, 0, x_t, out=x)
            qc.qconv2d_forward(d, x, w, b, mm, nn, y=y)

        for _ in range(args.warmup):
            launch()
        times = []
        for _ in range(args.steps):
            flush.fill_(i & 0xFF)
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            launch()
            e1.record()
            times.append((e0, e1))
        torch.cuda.synchronize()
        us = statistics.median(a.elapsed_time(z) * 1e3 for a, z in times)
        ops, nbytes = layer_algorithmic(cs, bits)
        if xf is not None:
            nbytes += cs.n * cs.h * cs.w * cs.c * (4 + bits / 8)
        roof = roofline_us(ops, nbytes, peaks)
        total_ops += ops
        total_us += us
        total_roof += roof
        # parity on one sampled image (the last) against the oracle
        img = cs.n - 1
        xs = x[img:img + 1].cpu().numpy()
        mo, no = oracle.requant_params(lp.s_x, lp.s_w, lp.s_y)
        ref = oracle.conv2d(xs, lp.w_bytes, n=1, h=cs.h, wd=cs.w, c=c_st, k=cs.k, r=cs.r, s=cs.s,
                            xt=x_t, wt=w_t, yt=x_t, stride=(cs.stride, cs.stride), pad=(cs.pad, cs.pad),
                            clamp_lo=lp.clamp_lo, clamp_hi=lp.clamp_hi, bias=lp.bias, mult=mo, shift=no)
        if not np.array_equal(y[img:img + 1].cpu().numpy(), ref):
            bad.append(cs.name)
        results.append({"name": cs.name, "n": cs.n, "us": us, "tops": ops / us / 1e6,
                        "gbs": nbytes / us / 1e3, "roofline_us": roof, "frac_roofline": roof / us,
                        "frac_tensor": ops / us / 1e6 / peaks["int8_tops"],
                        "kernel": plan["kernel_name"], "bn": plan["bn"]})
    clocks = clk.stop()
    if args.workload in ("c1", "c2"):
        r0 = results[0]
        value, unit, hib = r0["us"], "us per invocation (latency, cold L2)", False
        metric = "single-layer latency (BASELINE configs[%d])" % (0 if args.workload == "c1" else 1)
    elif args.workload == "c4":
        value, unit, hib = shapes[0].n / (total_us / 1e6), "images/s", True
        metric = "VGG-16 conv stack images/s (BASELINE configs[3])"
    else:
        value, unit, hib = total_ops / total_us / 1e6, "TOPS", True
        metric = f"per-layer conv TOPS ({args.workload})"
    line = {"metric": metric, "value": value, "unit": unit, "higher_is_better": hib,
            "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
            "dtype": f"int{bits} (int8 tcgen05 MMA, int32 acc)", "data": "synthetic (seeded)",
            "config": {"workload": args.workload, "layers": len(shapes), "bits": bits,
                       "l2": "flushed (512 MB write) before every timed launch",
                       "plans": "autotuned" if args.tune else "default rule"},
            "tops": total_ops / total_us / 1e6,
            "roofline": {"bound": "tensor", "achieved": total_ops / total_us / 1e6,
                         "peak": peaks["int8_tops"], "unit": "TOPS",
                         "frac": total_ops / total_us / 1e6 / peaks["int8_tops"],
                         "frac_of_roofline_time": total_roof / total_us,
                         "peak_source": peaks["source"]},
            "parity": {"sampled": "last image of every layer", "bit_exact": not bad, "mismatch": bad},
            "clocks": clocks, "layers": results}
    print(json.dumps(line), flush=True)
    if args.layers_json:
        with open(args.layers_json, "w") as f:
            json.dump(line, f, indent=1)
    if args.save_plans and tuned:
        from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning
        tuning.save_plans(args.save_plans, tuned, {"workload": args.workload, "bits": bits})
    return 0


# ----------------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--bits", type=int, default=4, choices=(4, 8))
    ap.add_argument("--workload", default="trunk", choices=("trunk", "c1", "c2", "c3", "c4", "f4"))
    ap.add_argument("--global-batch", type=int, default=GLOBAL_BATCH,
                    help="C5: total images, sharded over the GPUs (strong scaling)")
    ap.add_argument("--batch", type=int, default=0, help="weak scaling: images per GPU")
    ap.add_argument("--impl", default="ours", choices=("ours", "reference"))
    ap.add_argument("--tune", action="store_true", help="profile-run tile search before timing")
    ap.add_argument("--plans", default="", help="tile-search table to apply ('' = plans/<workload>.json "
                                                "if present, 'none' = the default rule)")
    ap.add_argument("--save-plans", default="", help="write the --tune results to this table")
    ap.add_argument("--stem-dtype", default="bf16", choices=("bf16", "fp32"),
                    help="dtype of the image the stem quantizes (and of the e2e H2D copy)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-verify", action="store_true")
    ap.add_argument("--layers-json", default="")
    ap.add_argument("--profile-steps", type=int, default=0,
                    help="only run warmup + N eager steps (for ncu), no JSON")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if args.workload != "trunk":
        return run_layers(args)
    return run_trunk(args)


if __name__ == "__main__":
    sys.exit(main())
