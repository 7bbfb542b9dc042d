#!/usr/bin/env python
"""TeMCO fused reduced-skip inference benchmark (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config resnet50] [--impl reference]

One step = one full forward pass (every schedule step of the TeMCO plan: core
convs, fused restore->BN->add->ReLU->reduce groups, head) over one per-GPU batch
of synthetic images already resident in HBM.  Under torchrun each rank runs its
own contiguous shard of the global batch (weak scaling) and the fp32 logits are
gathered with one NCCL all_gather per step (the only collective).
Rank 0 prints ONE JSON line.

`--impl reference` times the oracle (oracle/, fp64 numpy) as it stands on the
host cores -- the reference arm of this tier -- on a bounded sample per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

CONFIG_BATCH = {"resnet18_cifar": 128, "resnet50": 256, "vgg16_cp": 256, "densenet121": 128, "alexnet": 256, "unet": 16,
                "resnet18_tt": 128}
CONFIG_TEXT = {
    "resnet18_cifar": "ResNet-18 Tucker-2 decomposed, CIFAR-10 shape 32x32, batch 128",
    "resnet50": "ResNet-50 Tucker-2 decomposed, ImageNet shape 224x224, batch 256 per GPU, bf16",
    "vgg16_cp": "VGG-16 CP-decomposed convs, 224x224, batch 256 per GPU",
    "densenet121": "DenseNet-121 Tucker-2 decomposed (concat skips), 224x224, batch 128 per GPU, 8-GPU batch shard",
    "alexnet": "AlexNet Tucker-2 decomposed (SURVEY 8(f) f2; not a BASELINE.json config), 224x224, batch 256 per GPU",
    "unet": "UNet Tucker-2 decomposed (SURVEY 8(f) f1; Carvana shape 256x256, 2 classes; not a BASELINE.json config), batch 16 per GPU",
    "resnet18_tt": "ResNet-18 Tensor-Train decomposed K x K convs (SURVEY 8(f) f4; not a BASELINE.json config), CIFAR-10 shape 32x32, batch 128",
}
METRIC = "images/sec"


def _peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return d["hbm_gbs"], d["bf16_tflops"], d.get("bf16_tflops_sustained", d["bf16_tflops"]), "measured"
    return 6650.0, 1590.0, 1400.0, "fallback"


class Clocks:
    """SM clock and throttle reasons sampled DURING the timed region (B200_PROFILING.md clocks
    line): an NVML sampler thread every 2 ms (short steps end before nvidia-smi's 100 ms loop
    takes a sample); nvidia-smi -lms 100 as the fallback when NVML is unavailable."""

    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))

    def __init__(self, index):
        self.rows, self.p, self.t = [], None, None
        try:
            import threading

            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            self.stop_ev = threading.Event()

            def run():
                while not self.stop_ev.is_set():
                    try:
                        self.rows.append((pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM),
                                          pynvml.nvmlDeviceGetUtilizationRates(h).gpu,
                                          pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)))
                    except Exception:
                        pass
                    self.stop_ev.wait(0.002)

            self.t = threading.Thread(target=run, daemon=True)
            self.t.start()
            return
        except Exception:
            self.t = None
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("clocks.sm,clocks.max.sm,utilization.gpu,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(index), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "100"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.t is not None:
            self.stop_ev.set()
            self.t.join()
            if not self.rows:
                return None
            loaded = [r for r in self.rows if r[1] > 0] or self.rows
            reasons = sorted({n for r in loaded for n, bit in self.REASONS if r[2] & bit})
            return {"sm_mhz": statistics.median(r[0] for r in loaded), "sm_max_mhz": self.max_mhz,
                    "reasons": reasons, "samples": len(loaded), "source": "nvml"}
        if self.p is None:
            return None
        self.p.terminate()
        self.p.wait()
        rows = []
        for line in open(self.f.name):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7 and parts[0].isdigit():
                rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return None
        loaded = [r for r in rows if r[2].isdigit() and int(r[2]) > 0] or rows
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in loaded for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(int(r[0]) for r in loaded), "sm_max_mhz": int(rows[0][1]),
                "reasons": reasons, "samples": len(loaded), "source": "nvidia-smi"}


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def reference_arm(args):
    """Oracle (fp64 numpy) on the host cores: each step = a bounded sample."""
    import oracle
    ws, rank, _ = _dist()
    if rank != 0:
        return
    from threadpoolctl import threadpool_info
    m = W.build_config(args.config)
    sample = {"resnet18_cifar": 8, "resnet50": 1, "vgg16_cp": 1, "densenet121": 1, "alexnet": 1, "unet": 1,
              "resnet18_tt": 8}[args.config]
    pl = oracle.plan(m)
    times = []
    for step in range(args.warmup + args.steps):
        x = W.make_input(m, start=step * sample, count=sample)
        t0 = time.perf_counter()
        oracle.run_temco(pl, x)
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            times.append(dt)
    sec = sum(times) / len(times)
    value = sample / sec
    threads = max([t.get("num_threads", 1) for t in threadpool_info()] + [1])
    line = {"metric": METRIC, "value": value, "unit": "images/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": sec * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": args.config, "description": CONFIG_TEXT[args.config],
                       "sample_images_per_step": sample},
            "cpu_baseline": {"value": value, "unit": "images/s", "cores": threads, "kind": "oracle",
                             "sample": f"{sample} image(s) of {args.config} per step, TeMCO executor (fp64 numpy)"},
            "e2e": {"value": value, "unit": "images/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_baseline(config):
    """Oracle images/s on this host on ~10-30 s of CPU work (rank 0, N=1)."""
    import oracle
    from threadpoolctl import threadpool_info
    m = W.build_config(config)
    pl = oracle.plan(m)
    sample = {"resnet18_cifar": 256, "resnet50": 24, "vgg16_cp": 24, "densenet121": 24, "alexnet": 24, "unet": 4,
              "resnet18_tt": 256}[config]
    x = W.make_input(m, start=0, count=sample)
    oracle.run_temco(pl, x[:1])                 # warm-up
    t0 = time.perf_counter()
    oracle.run_temco(pl, x)
    dt = time.perf_counter() - t0
    threads = max([t.get("num_threads", 1) for t in threadpool_info()] + [1])
    return {"value": sample / dt, "unit": "images/s", "cores": threads, "kind": "oracle",
            "sample": f"{sample} images of {config} through the oracle's TeMCO executor (fp64 numpy), {dt:.1f} s"}


VARIANTS = {"temco": 0, "fusion_only": 2, "skipopt_only": 4, "decomposed": 6,   # TEMCO_FLAG_NO_SKIPOPT=2, NO_FUSION=4
            "paper_schedule": 1 << 9,   # the paper's schedule: no readings R34-R38 (TEMCO_FLAG_PAPER_SCHEDULE)
            "cse_bound": 1 << 12}       # reading R37 merges kept while the peak stays <= the unfused peak


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="resnet50", choices=list(CONFIG_BATCH))
    ap.add_argument("--impl", default="temco", choices=["temco", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--simt-only", action="store_true")
    # SURVEY 8(f) f3, the paper's ablations (Fig. 10/11) on the GPU:
    # decomposed = neither rewrite, fusion_only = no skip optimization,
    # skipopt_only = no fusion.  Not the headline line: same metric, other plan.
    ap.add_argument("--variant", default="temco", choices=list(VARIANTS))
    # the same network with every ReLU replaced by SiLU
    ap.add_argument("--act", default="relu", choices=["relu", "silu"])
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # `bench.py --gpus N` outside torchrun: launch N ranks (one process per GPU) on this
        # node through torch.distributed.run; rank 0 prints the line, the exit code is theirs
        env = dict(os.environ)
        env.setdefault("NCCL_DEBUG", "INFO")           # NCCL init lines (nranks) for the record
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={29500 + os.getpid() % 1000}",
               os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd, env=env)
    ws_env = int(os.environ.get("WORLD_SIZE", "1"))
    if ws_env != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws_env}")
    if args.impl == "reference":
        return reference_arm(args)

    import torch
    import torch.distributed as dist
    from paper_conf_icpp_songljkj0024_b200 import FLAG_CUDA_GRAPH, FLAG_SIMT_ONLY, Plan
    from paper_conf_icpp_songljkj0024_b200.shard import gather_logits, shard_range

    ws, rank, local = _dist()
    torch.cuda.set_device(local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    B = CONFIG_BATCH[args.config]
    m = W.build_config(args.config, batch=B)
    if args.act == "silu":
        for layer in m.layers:
            if layer.op == "relu":
                layer.op = "silu"
    flags = FLAG_CUDA_GRAPH | (FLAG_SIMT_ONLY if args.simt_only else 0) | VARIANTS[args.variant]
    plan = Plan(m, flags=flags)
    desc = plan.describe()
    out_shape = plan.output_shape()
    start, stop = shard_range(rank, ws, B)
    x_host = W.make_input(m, start=start, count=stop - start)
    tdt = torch.bfloat16 if m.dtype == "bf16" else torch.float32
    x = torch.from_numpy(x_host).to(tdt).cuda()
    y = torch.empty(out_shape, dtype=torch.float32, device="cuda")
    gathered = torch.empty((ws,) + tuple(out_shape), dtype=torch.float32, device="cuda") if ws > 1 else None
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")      # > 126 MB L2
    stream = torch.cuda.Stream()

    def step():
        plan.run(x, y, stream)
        if ws > 1:
            gather_logits(y, ws, gathered)

    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            step()
    torch.cuda.synchronize()

    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    clocks = Clocks(local)
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        for i in range(args.steps):
            flush.fill_(i & 0xFF)                                            # L2 flush, outside the events
            evs[i][0].record(stream)
            step()
            evs[i][1].record(stream)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = sum(a.elapsed_time(b) for a, b in evs)
    if ws > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_per_step = ms / args.steps
    value = ws * B / (ms_per_step / 1e3)

    # ---- end to end through the public API with host buffers -----------------
    # temco_run_host_async: every step copies its input host->device (pinned,
    # on the plan's copy stream, overlapping the previous step's compute), runs,
    # and copies the logits back; the region ends after the last D2H completes
    xh = torch.from_numpy(x_host).to(tdt).pin_memory()
    yh = torch.empty(out_shape, dtype=torch.float32).pin_memory()
    plan.run_host(xh, yh, stream)
    plan.run_host_async(xh, yh, stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if ws > 1:
        dist.barrier()
    e0.record(stream)
    with torch.cuda.stream(stream):
        for _ in range(args.steps):
            plan.run_host_async(xh, yh, stream)
            if ws > 1:
                # this step's logits (host) back on the device for the NCCL gather, stream-ordered
                y.copy_(yh, non_blocking=True)
                gather_logits(y, ws, gathered)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1) / args.steps
    if ws > 1:
        t = torch.tensor([e2e_ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())

    # ---- roofline of the dominant kernel class (per-step CUDA events) --------
    steps = desc["steps"]
    prof = np.zeros(len(steps))
    n_prof = max(3, min(args.steps, 10))
    with torch.cuda.stream(stream):
        for _ in range(n_prof):
            flush.fill_(1)
            prof += np.array(plan.run_profiled(x, y, stream))
    prof /= n_prof
    classes = {}
    for s, t in zip(steps, prof):
        k = s["kernel"]
        if s["launches"] == 0:      # "none" (the input) and steps produced by another step's epilogue
            continue
        c = classes.setdefault(k, {"ms": 0.0, "flops": 0, "bytes": 0, "launches": 0})
        c["ms"] += float(t)
        c["flops"] += s.get("alg_flops", s["flops"])
        c["bytes"] += s.get("alg_bytes", s["io_bytes"])
        c["launches"] += s["launches"]
    hbm, tf_burst, tf_sust, src = _peaks()
    # per-step event timing breaks the graph / programmatic-launch overlap and inflates the
    # sum (~+14 %): class times are its SHARES scaled to the graph-run step time
    total_ms = float(prof.sum())
    scale = ms_per_step / total_ms if total_ms > 0 else 1.0
    for v in classes.values():
        v["ms_events"] = v["ms"]
        v["ms"] = v["ms"] * scale
    # burst bf16 peak when the SM clock held its maximum during the timed region (the
    # sustained figure is cuBLAS under the power cap at ~1.3 GHz), else sustained
    at_max = bool(clk and clk.get("sm_max_mhz") and clk["sm_mhz"] >= 0.97 * clk["sm_max_mhz"])
    tf_peak = tf_burst if at_max else tf_sust
    dom = max(classes, key=lambda k: classes[k]["ms"])
    c = classes[dom]
    ai = c["flops"] / max(c["bytes"], 1)
    if ai > tf_peak * 1e12 / (hbm * 1e9):
        achieved, peak, unit, bound = c["flops"] / (c["ms"] * 1e-3) / 1e12, tf_peak, "TFLOP/s", "tensor"
    else:
        achieved, peak, unit, bound = c["bytes"] / (c["ms"] * 1e-3) / 1e9, hbm, "GB/s", "hbm"
    total_ms = ms_per_step
    # every class against its own bound, and the fused-group family (SURVEY 8(a)
    # row a6: tc_chain + mma_lean + mma_chain) as a time-weighted roofline
    # fraction over its launches (+ mma_poolcat / mma_cat): sum_i max(F_i / P_tc, B_i / P_hbm) / sum_i t_i
    by_class = {}
    for k, v in classes.items():
        a_i = v["flops"] / max(v["bytes"], 1)
        tb = a_i > tf_peak * 1e12 / (hbm * 1e9)
        ach = v["flops"] / (v["ms"] * 1e-3) / 1e12 if tb else v["bytes"] / (v["ms"] * 1e-3) / 1e9
        by_class[k] = {"bound": "tensor" if tb else "hbm", "achieved": round(ach, 1),
                       "unit": "TFLOP/s" if tb else "GB/s", "frac": round(ach / (tf_peak if tb else hbm), 4),
                       "ms": round(v["ms"], 4)}
    fused_k = ("tc_pair", "tc_chain", "tc_chain_wide", "mma_lean", "mma_chain", "mma_poolcat", "mma_cat", "mma_catp")
    ideal = actual = 0.0
    for s, t in zip(steps, prof):
        if s["kernel"] in fused_k and t > 0:
            ideal += max(s.get("alg_flops", s["flops"]) / (tf_peak * 1e12), s.get("alg_bytes", s["io_bytes"]) / (hbm * 1e9))
            actual += float(t) * scale * 1e-3
    fused = {"kernels": list(fused_k), "roofline_ms": round(ideal * 1e3, 4),
             "measured_ms": round(actual * 1e3, 4), "frac": round(ideal / actual, 4) if actual else None,
             "note": "per launch max(alg FLOP / bf16 peak, alg bytes / HBM peak), summed, / measured (graph-run share)"}
    # DRAM traffic of the dominant class from the committed ncu capture of this
    # config (scripts/launch_summary.py --json), bytes per step like `achieved`
    traffic = None
    tpath = os.path.join(ROOT, "profiles", f"traffic_{args.config}.json")
    if os.path.exists(tpath) and args.variant == "temco":
        traffic = json.load(open(tpath)).get(dom)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "images/s", "per_gpu_value": value / ws,
            "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": m.dtype, "data": "synthetic",
            "config": {"workload": args.config, "description": CONFIG_TEXT[args.config], "batch_per_gpu": B,
                       "global_batch": ws * B, "image_hw": [m.height, m.width], "parallelism": f"dp{ws}",
                       "l2": "flushed between timed steps (512 MiB write, outside the step events)",
                       "peak_internal_bytes": plan.peak_internal_bytes(0),
                       "peak_internal_bytes_unfused": plan.peak_internal_bytes(1),
                       "internal_memory_reduction": 1 - plan.peak_internal_bytes(0) / plan.peak_internal_bytes(1),
                       "cuda_graph": True, "kernels": "simt-only" if args.simt_only else "tcgen05+simt",
                       "variant": args.variant, "activation": args.act},
            "gpu_launches": desc["launches"] * args.steps,
            "e2e": {"value": ws * B / (e2e_ms / 1e3), "unit": "images/s", "api": "temco_run_host_async (pipelined H2D)",
                    "h2d_bytes_per_step": int(xh.numel() * xh.element_size()),
                    "d2h_bytes_per_step": int(yh.numel() * yh.element_size())},
            "roofline": {"bound": bound, "kernel": dom, "achieved": achieved, "peak": peak, "unit": unit,
                         "frac": achieved / peak, "traffic": traffic,
                         "traffic_note": "DRAM read+write bytes per step of the class (ncu, cold L2), from "
                                         "profiles/traffic_<config>.json", "peak_source": src,
                         "peak_kind": "burst (SM clock at max)" if at_max else "sustained",
                         "time_source": "per-step CUDA-event shares x graph-run ms/step",
                         "launches_per_step": c["launches"], "share_of_step": c["ms"] / total_ms,
                         "alg_flops_per_step": c["flops"], "alg_bytes_per_step": c["bytes"]},
            "kernel_classes_ms": {k: round(v["ms"], 4) for k, v in sorted(classes.items(), key=lambda kv: -kv[1]["ms"])},
            "roofline_by_class": by_class,
            "fused_group_roofline": fused,
            "clocks": clk,
        }
        if ws == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(args.config)
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
