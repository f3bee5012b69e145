#!/usr/bin/env python
"""PASK on B200 -- benchmark driver (one JSON line on rank 0).

Workload (BASELINE.json configs[1]): ResNet-50, batch 1, 224x224, bf16, random
weights, synthetic N(0,1) input.  A "step" is one inference through the C ABI
(pask_infer: all 58 layers).  Metric (BASELINE.json): cold first-inference
latency vs hot; imgs/s per B200; kernels loaded per model.

  value  imgs/s over all ranks = N * batch * 1000 / max-over-ranks(hot ms), hot =
         K timed inferences replaying the captured CUDA graph, L2 flushed before
         each (a 256 MiB memset outside the CUDA-event window)
  cold   SURVEY.md §8(d): >= 20 fresh native processes (pask_cold), each
         t0 = pask_load_model entry -> t1 = first inference done; median / p90,
         with and without the host prefault of the code images, and a timeline
         set (cfg.timeline: per-kernel %globaltimer stamps) for the partitioned
         breakdown (Fig. 1(b) / Fig. 7) and the cold GPU utilisation (Fig. 6(b))
  hot    graph replay (value) and direct issue (the cold start's own issue
         path without loading: the paper's Ideal)
  packaging 3 (default, D15): the cold start uploads one function
         (pask_all of the model's variant); after it, in the idle interval,
         pask_promote repacks the model into the two family entries, which the
         hot inferences run on (cold children: pask_cold --promote before --hot)
  e2e    pask_infer_host: pinned host input -> H2D -> the model -> D2H of the
         outputs -> sync, host clock per step
  headline  the LAST key of the line: the compact cold / hot / ratio / util /
         breakdown / kernels block of every config (C1-C4) from this run

N > 1 (torchrun): independent replicas, one process per GPU (SURVEY.md §8(e):
the path does not shard; no data-path collective -- gloo carries the barrier,
the max and the gather of the replica statistics).  Every rank cold-starts
native pask_cold children released together after a barrier (>= 10 trials),
then rank 0 alone for the same-run cold(1) -> loader contention cold(N)/cold(1).

`--impl reference` times the fp64 numpy oracle (the reference arm of this
tier) on the host cores, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "cold first-inference latency ms vs hot; imgs/s per B200; kernels loaded/model"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}
CONFIG_MODELS = ["tiny_cnn", "resnet50", "mobilenet_v2", "bert_base"]   # BASELINE.json configs[0..3]
BREAKDOWN_KEYS = ["plan", "load", "issue", "gpu_busy", "gpu_idle", "other"]


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return PEAKS_FALLBACK, "fallback"


# ---------------------------------------------------------------- algorithmic work
def node_work(spec, li):
    """(bytes, flops) of layer li: bytes = inputs + weights +
    outputs (+ residual, bias, gamma / beta) at their device precision (bf16
    tensors, fp32 vectors; the stem reads its input padded to 8 channels, which
    the kernel really moves); flops = 2 x the multiply-adds of the logical
    operator (unpadded channels)."""
    L = spec["layers"][li]
    sh = spec["tensors"]
    op = L["op"]

    def numel(name):
        n = 1
        for d in sh[name]:
            n *= d
        return n
    if op == "layout":
        n, c, h, w = sh[L["inputs"][0]]
        return n * c * h * w * 4 + n * h * w * L["c_pad"] * 2, 0
    if op == "conv":
        k, cg, r, s = L["w"].shape
        n, c, h, w = sh[L["inputs"][0]]
        dense = L["groups"] == 1
        c_dev = max(8, (c + 7) // 8 * 8) if dense else c
        _, _, p, q = sh[L["out"]]
        byt = n * h * w * c_dev * 2 + k * r * s * (c_dev if dense else 1) * 2 + \
            n * p * q * k * 2 + (k * 4 if L["b"] is not None else 0)
        if L["res"]:
            byt += n * p * q * k * 2
        return byt, 2 * n * p * q * k * cg * r * s
    if op == "linear":
        m, nout = sh[L["out"]]
        kin = L["w"].shape[1]
        byt = m * kin * 2 + nout * kin * 2 + m * nout * 2 + (nout * 4 if L["b"] is not None else 0)
        if L["res"]:
            byt += m * nout * 2
        return byt, 2 * m * nout * kin
    if op == "qk":     # scores[h] = Q_h K_h^T: read Q and K, write the scores
        heads, dh = L["heads"], L["head_dim"]
        s_ = sh[L["inputs"][0]][0]
        return 2 * s_ * heads * dh * 2 + heads * s_ * s_ * 2, 2 * heads * s_ * s_ * dh
    if op == "pv":     # ctx[:, h] = P_h V_h: read P and V, write the context
        heads, dh = L["heads"], L["head_dim"]
        s_ = sh[L["inputs"][1]][0]
        return heads * s_ * s_ * 2 + s_ * heads * dh * 2 + s_ * heads * dh * 2, 2 * heads * s_ * dh * s_
    if op == "attention":   # fused: read Q, K, V, write the context
        heads, dh = L["heads"], L["head_dim"]
        s_ = sh[L["inputs"][0]][0]
        return 3 * s_ * heads * dh * 2 + s_ * heads * dh * 2, 4 * heads * s_ * s_ * dh
    if op == "layernorm":
        cols = sh[L["inputs"][0]][-1]
        return numel(L["inputs"][0]) * 2 + numel(L["out"]) * 2 + 2 * cols * 4, 0
    return numel(L["inputs"][0]) * 2 + numel(L["out"]) * 2, 0   # pool, softmax


def step_shares(intervals, kernels):
    """Partition of one inference's GPU busy time among the catalog solutions,
    from the timeline stamps of a PDL-chained (graph-replayed) step: in end-time
    order, node i is charged end_i - max(start_i, latest end before it), the
    time during which it was the last node to finish.  Charges sum to the busy
    union.  Returns {kernel: (charged_ns, launches)}."""
    order = sorted(range(len(intervals)), key=lambda i: intervals[i][1])
    out, latest = {}, None
    for i in order:
        s, e = intervals[i]
        if e == 0 and s == 0:
            continue
        lo = s if latest is None else max(s, latest)
        ch = max(0, e - lo)
        latest = e if latest is None else max(latest, e)
        c, n = out.get(kernels[i], (0, 0))
        out[kernels[i]] = (c + ch, n + 1)
    return out


# ---------------------------------------------------------------- replicas
def reduce_max(values, dist=None):
    """Element-wise max over ranks (gloo all_reduce on CPU; no data-path
    collective: replicas share nothing but this timing reduction)."""
    import torch
    t = torch.tensor([float(v) for v in values], dtype=torch.float64)
    if dist is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t]


def replica_cold_trials(run_waiting_child, dist, rank, trials):
    """`trials` concurrent cold starts -- every rank starts its
    child (set up, waiting), a barrier, then each releases its child into the
    cold window -- and `trials` solo cold starts of rank 0 (the others wait at
    the barrier) for the same-run cold(1).  run_waiting_child() returns
    (release, collect): release() lets the child start its cold window,
    collect() returns its JSON result.  Returns (concurrent, solo) lists of
    result dicts (solo empty on ranks != 0)."""
    conc, solo = [], []
    for _ in range(trials):
        release, collect = run_waiting_child()
        dist.barrier()
        release()
        conc.append(collect())
        dist.barrier()
    for _ in range(trials):
        if rank == 0:
            release, collect = run_waiting_child()
            release()
            solo.append(collect())
        dist.barrier()
    return conc, solo


def replica_summary(per_rank_conc, solo, per_rank_hot_ms, batch):
    """Rank 0's replica block: per-replica cold median / max over the trials,
    the contention ratio cold(N) / cold(1) (medians, same run), per-replica
    kernels loaded, and aggregate / per-GPU hot imgs/s."""
    n = len(per_rank_conc)
    per = []
    for r, trials in enumerate(per_rank_conc):
        c = [t["cold_us"] / 1e3 for t in trials]
        per.append({"rank": r, "cold_med_ms": round(statistics.median(c), 3), "cold_max_ms": round(max(c), 3),
                    "trials": len(c), "kernels_loaded": sorted({int(t["kernels_loaded"]) for t in trials}),
                    "cold_ms": [round(v, 3) for v in c]})
    all_conc = [t["cold_us"] / 1e3 for trials in per_rank_conc for t in trials]
    solo_ms = [t["cold_us"] / 1e3 for t in solo]
    cn = statistics.median(all_conc)
    c1 = statistics.median(solo_ms) if solo_ms else None
    agg = sum(batch * 1000.0 / h for h in per_rank_hot_ms)
    return {"n_replicas": n, "cold_N_med_ms": round(cn, 3), "cold_N_max_ms": round(max(all_conc), 3),
            "cold_1_med_ms": round(c1, 3) if c1 else None,
            "contention": round(cn / c1, 3) if c1 else None,
            "per_replica": per, "hot_imgs_s_aggregate": round(agg, 1),
            "hot_imgs_s_per_gpu": round(agg / n, 1)}


# ---------------------------------------------------------------- clocks
class ClockSampler:
    def __init__(self, device):
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "50", "-i", str(device)],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------- reference arm / cpu baseline
def time_oracle(spec, x, max_steps, budget_s):
    """The fp64 numpy oracle, as it stands, full forwards of one image."""
    from oracle import models as om
    times = []
    t_end = time.perf_counter() + budget_s
    for _ in range(max_steps):
        t0 = time.perf_counter()
        om.run_model(spec, x)
        times.append(time.perf_counter() - t0)
        if time.perf_counter() > t_end:
            break
    return times


def cores_used():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count()


def cpu_model():
    """The host CPU's model name (state the CPU the oracle ran on)."""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def run_reference(args, spec, x, rank):
    if rank != 0:
        return
    w = time_oracle(spec, x, max(args.warmup, 0), 60.0) if args.warmup else []
    ts = time_oracle(spec, x, args.steps, 240.0)
    mean_s = statistics.mean(ts)
    val = args.batch / mean_s
    line = {
        "impl": "reference", "metric": METRIC, "value": round(val, 4), "unit": "imgs/s",
        "n_gpus": args.gpus, "steps": len(ts), "warmup": len(w), "ms_per_step": round(1e3 * mean_s, 2),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": {"workload": args.workload_name, "global_batch": args.batch,
                                        "model": args.model},
        "cpu_baseline": {"value": round(val, 4), "unit": "imgs/s", "cores": cores_used(),
                         "kind": "oracle", "cpu": cpu_model(),
                         "sample": f"{len(ts)} full fp64 numpy-oracle forwards of a batch-{args.batch} input"},
        "e2e": {"value": round(val, 4), "unit": "imgs/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- cold samples (native children)
def bench_cfg(args, **extra):
    return {"packaging": args.packaging, "branches": args.branches, "graph": args.graph, **extra}


def cold_block(cs, image, cfg, n, n_tl, hot_children):
    """Fresh-process cold samples of one config: n cold starts, n_tl timeline
    cold starts (breakdown + utilisation), and optionally hot children (graph
    replay and direct issue, L2 flushed, 200 inferences each)."""
    samples = cs.sample(image, cfg, n)
    tl = cs.sample(image, {**cfg, "timeline": 1}, n_tl) if n_tl else []
    out = {"cold": cs.summarize(samples), "breakdown": cs.breakdown(tl) if tl else None,
           "plan": [samples[0]["queries"], samples[0]["hits"], samples[0]["lookups"]],
           "launches": samples[0]["launches"], "load_timeline_us": samples[0]["timeline"]}
    if tl:
        out["cold_timeline_med_us"] = statistics.median(s["cold_us"] for s in tl)
    if hot_children:
        out["hot_graph_us"] = cs.run_child(image, {**cfg, "graph": 1}, hot=200)["hot_median_us"]
        out["hot_direct_us"] = cs.run_child(image, {**cfg, "graph": 0}, hot=200)["hot_median_us"]
    return out


def headline_entry(cold_ms, p90_ms, n, hot_graph_ms, hot_direct_ms, bd, kernels, launches, extra=None):
    e = {"cold_ms": [round(cold_ms, 3), round(p90_ms, 3), n],
         "hot_ms": [round(hot_graph_ms, 4), round(hot_direct_ms, 4)],
         "cold/hot": [round(cold_ms / hot_graph_ms, 2), round(cold_ms / hot_direct_ms, 2)],
         "util": bd["util"] if bd else None,
         "bd_us": [round(bd[k]) for k in BREAKDOWN_KEYS] if bd else None,
         "kernels": int(kernels), "launches": int(launches)}
    if extra:
        e.update(extra)
    return e


# ---------------------------------------------------------------- main
_T0 = time.time()


def phase(msg):
    """Progress on stderr (the JSON line is the only stdout)."""
    print(f"[bench {time.time() - _T0:7.1f}s] {msg}", file=sys.stderr, flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="pask", choices=["pask", "reference"])
    ap.add_argument("--model", default="resnet50",
                    choices=["tiny_cnn", "resnet50", "mobilenet_v2", "bert_base", "bert_base_fa"])
    ap.add_argument("--batch", type=int, default=1, help="images per inference (Table II sweep)")
    ap.add_argument("--branches", type=int, default=1, choices=[0, 1],
                    help="1 (default): independent nodes (ResNet downsample convs) on a second stream "
                         "(DESIGN.md D9)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cold-samples", type=int, default=20,
                    help="fresh-process cold starts per config (native pask_cold children)")
    ap.add_argument("--timeline-samples", type=int, default=10,
                    help="fresh-process cold starts with cfg.timeline (breakdown, GPU utilisation)")
    ap.add_argument("--ablation-samples", type=int, default=10,
                    help="fresh processes for the no-prefault / no-primer ablations of the main config")
    ap.add_argument("--py-cold-samples", type=int, default=5,
                    help="main config: cold starts in fresh PyTorch processes (framework process state)")
    ap.add_argument("--no-configs", action="store_true",
                    help="skip the other configs' compact block (C1-C4 headline)")
    ap.add_argument("--replica-trials", type=int, default=10, help="N > 1: concurrent cold-start trials")
    ap.add_argument("--no-flush", action="store_true", help="L2-warm hot loop (reported as such)")
    ap.add_argument("--graph", type=int, default=1, choices=[0, 1],
                    help="1: hot inferences replay a CUDA graph captured on the 2nd call")
    ap.add_argument("--packaging", type=int, default=3, choices=[0, 1, 2, 3],
                    help="0: one code object per catalog kernel; 1: whole catalog in one; "
                         "2: operator families, DESIGN.md D8; 3 (default): single function for the "
                         "cold start, repacked into the families after it (D10, D15)")
    args = ap.parse_args()
    args.workload_name = {
        "tiny_cnn": "tiny CNN 3xconv3x3(16/32/64)+maxpool+FC, 32x32x3, batch 1, bf16",
        "resnet50": "ResNet-50 batch 1 224x224 cold start, all convs served by one reused "
                    "implicit-GEMM kernel",
        "mobilenet_v2": "MobileNetV2 batch 1 224x224 (depthwise + pointwise convs) cold start",
        "bert_base": "BERT-base seq 128 batch 1 (GEMM + softmax + layernorm) cold start",
        "bert_base_fa": "BERT-base seq 128 batch 1 cold start, attention fused (QK^T -> softmax -> PV "
                        "in one kernel; SURVEY.md 8(f) NEXT #4)",
    }[args.model]
    if args.batch != 1:
        args.workload_name += f" (Table II sweep: batch {args.batch})"

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    dist = None
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("gloo", rank=rank, world_size=world)

    from workloads import build_model
    spec, x = build_model(args.model, **({"batch": args.batch} if args.batch != 1 else {}))

    if args.impl == "reference":
        run_reference(args, spec, x, rank)
        if dist:
            dist.destroy_process_group()
        return

    import torch

    from paper_conf_dac_huangdxz25_b200 import build as pbuild
    from paper_conf_dac_huangdxz25_b200 import pask as P
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from scripts import cold_samples as cs

    pbuild.build()

    # ---------------- cold in fresh native processes (N = 1; with replicas the
    # concurrent trials below are the measurement), taken BEFORE this process
    # creates its CUDA context.  An idle keeper process holds a context
    # meanwhile (the GPU stays initialised between children, as under a
    # persistence daemon; cold medians unchanged, r3h_keeper.log)
    main_cold, configs_detail = None, {}
    if world == 1 and args.cold_samples > 0:
        phase("cold samples: " + args.model)
        cfg = bench_cfg(args)
        image = cs.write_image(args.model, batch=args.batch)
        try:
            with cs.Keeper(image, cfg):
                main_cold = cold_block(cs, image, cfg, args.cold_samples, args.timeline_samples, False)
                if args.ablation_samples > 0:
                    main_cold["cold_no_prefault"] = cs.summarize(cs.sample(image, {**cfg, "no_prefault": 1},
                                                                           args.ablation_samples))
                    main_cold["cold_no_prime"] = cs.summarize(cs.sample(image, {**cfg, "no_prime": 1},
                                                                        args.ablation_samples))
                py = [cs.run_py_child(args.model, cfg, args.batch) for _ in range(args.py_cold_samples)]
                main_cold["cold_python_process"] = cs.summarize(py) if py else None
                if not args.no_configs and args.batch == 1:
                    for m in CONFIG_MODELS:
                        if m == args.model:
                            continue
                        phase("cold samples: " + m)
                        img_m = cs.write_image(m)
                        try:
                            configs_detail[m] = cold_block(cs, img_m, cfg, args.cold_samples,
                                                           args.timeline_samples, True)
                        finally:
                            os.unlink(img_m)
        finally:
            os.unlink(image)

    # one replica per GPU (LOCAL_RANK -> device); on a box with fewer GPUs than
    # ranks (a harness check on one GPU) ranks share devices round-robin
    phase("hot measurement")
    local_rank = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    stream = torch.cuda.current_stream(dev)
    sp = stream.cuda_stream
    dm = DeviceModel(spec, device=dev)
    dm.set_input(x)
    flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def flush():
        flush_buf.zero_()

    flush()
    torch.cuda.synchronize()
    ctx = P.Context(local_rank, P.config(packaging=args.packaging, graph=args.graph, branches=args.branches))
    n_nodes = len(spec["layers"])

    def barrier():
        if dist:
            dist.barrier()

    # ---------------- in-process cold: pask_load_model entry -> first inference done
    barrier()
    torch.cuda.synchronize()
    ctx.load_model(dm.graph, plan=False)
    ctx.infer(sp)
    ctx.sync()
    plan = ctx.bindings()
    cold_stats = ctx.stats()
    cold_inproc_ms = cold_stats["cold_wall_ns"] / 1e6
    solutions = sorted(P.kernel_name(k) for k in {b[2] for b in plan})  # Algorithm 1's bound set
    loaded = sorted({P.function_name(k, args.packaging) for k in range(P.num_kernels())
                     if ctx.kernel_is_loaded(k)})                       # CUfunctions resident
    if args.packaging == 3:
        ctx.promote()   # idle interval after the cold start: repack into the family entries (D15)

    # ---------------- warmup
    for _ in range(args.warmup):
        flush()
        ctx.infer(sp)
    torch.cuda.synchronize()

    # ---------------- timed: K steps, L2 flushed between steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    sampler = ClockSampler(local_rank)
    time.sleep(0.2)
    barrier()
    torch.cuda.synchronize()
    w0 = time.perf_counter()
    for i in range(args.steps):
        if not args.no_flush:
            flush()
        ev[i][0].record(stream)
        ctx.infer(sp)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    w1 = time.perf_counter()
    barrier()
    clocks = sampler.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    hot_ms = statistics.mean(step_ms)
    hot_med_ms = statistics.median(step_ms)

    # ---------------- L2-warm back-to-back (context: serving the same model repeatedly)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    nw = max(20, args.steps // 2)
    for _ in range(nw):
        ctx.infer(sp)
    e1.record(stream)
    torch.cuda.synchronize()
    hot_warm_ms = e0.elapsed_time(e1) / nw

    # ---------------- e2e through the public API with host buffers
    (in_name, _, _), = spec["inputs"]
    in_host = torch.from_numpy(x.astype("float32")).to(dm.t[in_name].dtype).pin_memory()
    outs_host = [torch.empty(dm.t[o].shape, dtype=dm.t[o].dtype).pin_memory() for o in spec["outputs"]]
    h2d = in_host.numel() * in_host.element_size()
    d2h = sum(o.numel() * o.element_size() for o in outs_host)
    e2e_s = []
    for i in range(args.warmup + args.steps):
        if not args.no_flush:
            flush()
        torch.cuda.synchronize()
        a = time.perf_counter()
        ctx.infer_host([in_host.data_ptr()], [o.data_ptr() for o in outs_host], sp)
        b = time.perf_counter()
        if i >= args.warmup:
            e2e_s.append(b - a)
    e2e_ms = 1e3 * statistics.mean(e2e_s)

    # ---------------- hot through the direct-issue path (the paper's
    # "Ideal", PAPER.md:178 -- the cold start's own issue path without any loading),
    # L2 flushed like the timed loop; a separate context, graph off
    if args.graph:
        dctx = P.Context(local_rank, P.config(packaging=args.packaging, graph=0, branches=args.branches))
        dctx.load_model(dm.graph, plan=False)
        if args.packaging == 3:
            dctx.promote()
        for _ in range(args.warmup):
            flush()
            dctx.infer(sp)
        torch.cuda.synchronize()
        dev_ = []
        for i in range(args.steps):
            if not args.no_flush:
                flush()
            a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a_.record(stream)
            dctx.infer(sp)
            b_.record(stream)
            dev_.append((a_, b_))
        torch.cuda.synchronize()
        d_ms = [a_.elapsed_time(b_) for a_, b_ in dev_]
        hot_direct_ms = statistics.mean(d_ms)
        hot_direct_med_ms = statistics.median(d_ms)
        dctx.close()
    else:
        hot_direct_ms, hot_direct_med_ms = hot_ms, hot_med_ms

    # ---------------- per-kernel roofline: each solution's share of the step from
    # the timeline stamps of graph-replayed, PDL-chained steps (a separate context,
    # cfg.timeline), times the event-timed hot step
    tctx = P.Context(local_rank, P.config(packaging=args.packaging, graph=args.graph, branches=args.branches,
                                          timeline=1))
    tctx.load_model(dm.graph, plan=False)
    if args.packaging == 3:
        tctx.promote()
    kern_of = [b[2] for b in plan]
    charged = {}
    for r in range(12):
        flush()
        tctx.infer(sp)
        tctx.sync()
        if r >= 2:
            for k, (c, nl) in step_shares(tctx.node_intervals(), kern_of).items():
                cc, nn = charged.get(k, (0, 0))
                charged[k] = (cc + c, nn + nl)
    tctx.close()
    # ... and the isolated per-launch figure (events around each node, no PDL overlap)
    ictx = P.Context(local_rank, P.config(instrument=1))
    ictx.load_model(dm.graph)
    reps = 10
    acc = [0] * n_nodes
    for r in range(reps + 2):
        flush()
        ictx.infer(sp)
        ictx.sync()
        if r >= 2:
            acc = [a + b for a, b in zip(acc, ictx.node_times())]
    iso_ms = [a / reps / 1e6 for a in acc]
    ictx.close()
    per_kernel = {}
    for (i, want, bound, how, lk), t in zip(plan, iso_ms):
        byt, fl = node_work(spec, i)
        d = per_kernel.setdefault(bound, {"launches": 0, "iso_ms": 0.0, "bytes": 0, "flops": 0})
        d["launches"] += 1
        d["iso_ms"] += t
        d["bytes"] += byt
        d["flops"] += fl
    tot_charged = sum(c for c, _ in charged.values()) or 1
    for k, d in per_kernel.items():
        d["share"] = charged.get(k, (0, 0))[0] / tot_charged
        d["step_ms"] = d["share"] * hot_ms
    dom = max(per_kernel, key=lambda k: per_kernel[k]["step_ms"])
    peaks, peak_src = load_peaks()
    dk = per_kernel[dom]
    gbs = dk["bytes"] / (dk["step_ms"] * 1e-3) / 1e9
    tfl = dk["flops"] / (dk["step_ms"] * 1e-3) / 1e12
    gbs_iso = dk["bytes"] / (dk["iso_ms"] * 1e-3) / 1e9
    per_kernel_roofline = {}
    for k, v in per_kernel.items():
        st_ms = max(v["step_ms"], 1e-9)
        per_kernel_roofline[P.kernel_name(k)] = {
            "launches": v["launches"], "bytes_per_launch": int(v["bytes"] / v["launches"]),
            "in_step_us_per_launch": round(1e3 * st_ms / v["launches"], 2),
            "share": round(v["share"], 4),
            "achieved_gbs": round(v["bytes"] / (st_ms * 1e-3) / 1e9, 1),
            "frac_hbm": round(v["bytes"] / (st_ms * 1e-3) / 1e9 / peaks["hbm_gbs"], 4),
            "tflops": round(v["flops"] / (st_ms * 1e-3) / 1e12, 2),
            "isolated_us_per_launch": round(1e3 * v["iso_ms"] / v["launches"], 2)}
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "dram_traffic.json")
    if os.path.exists(tpath):
        with open(tpath) as f:
            traffic = json.load(f).get(args.model, {}).get(P.kernel_name(dom))
    roofline = {"bound": "hbm", "achieved": round(gbs, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": round(gbs / peaks["hbm_gbs"], 4), "traffic": traffic,
                "kernel": P.kernel_name(dom), "launches_per_step": dk["launches"],
                "algorithmic_bytes_per_launch": int(dk["bytes"] / dk["launches"]),
                "avg_launch_us": round(1e3 * dk["step_ms"] / dk["launches"], 2),
                "share_of_step": round(dk["share"], 4),
                "method": "achieved = algorithmic bytes / (share of the step x event-timed hot step); share = "
                          "the kernel's charge of the busy time in graph-replayed PDL steps (timeline stamps)",
                "isolated": {"avg_launch_us": round(1e3 * dk["iso_ms"] / dk["launches"], 2),
                             "achieved": round(gbs_iso, 1), "frac": round(gbs_iso / peaks["hbm_gbs"], 4),
                             "how": "events around each node, no PDL overlap (launch + prologue exposed)"},
                "tensor_tflops": round(tfl, 2),
                "tensor_frac_of_bf16_burst": round(tfl / peaks["bf16_tflops"], 4),
                "peak_source": f"{peak_src} (MEASURED_PEAKS.json hbm_gbs / bf16_tflops)",
                "l2": "flushed before each inference (weights from HBM)"}
    ctx.close()

    # ---------------- N > 1: concurrent replica cold starts (native children)
    replicas = None
    if world > 1:
        image = cs.write_image(args.model, batch=args.batch)
        cfg = bench_cfg(args)

        def waiting_child():
            p = subprocess.Popen([cs.EXE, image, "--cfg", cs.cfg_arg(cfg), "--device", str(local_rank),
                                  "--wait"], stdin=subprocess.PIPE, stdout=subprocess.PIPE,
                                 stderr=subprocess.PIPE, text=True)
            if p.stdout.readline().strip() != "ready":
                raise RuntimeError("replica child failed: " + p.stderr.read()[-2000:])

            def release():
                p.stdin.write("go\n")
                p.stdin.flush()

            def collect():
                so, se = p.communicate(timeout=120)
                return json.loads([l for l in so.splitlines() if l.startswith("{")][-1])
            return release, collect
        conc, solo = replica_cold_trials(waiting_child, dist, rank, args.replica_trials)
        os.unlink(image)
        gathered = [None] * world
        dist.all_gather_object(gathered, {"conc": conc, "solo": solo, "hot_ms": hot_ms})
        if rank == 0:
            replicas = replica_summary([g["conc"] for g in gathered], gathered[0]["solo"],
                                       [g["hot_ms"] for g in gathered], args.batch)

    # ---------------- max over ranks
    hot_max, e2e_max, warm_max, direct_max = reduce_max([hot_ms, e2e_ms, hot_warm_ms, hot_direct_ms], dist)
    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return

    # ---------------- headline: the fresh-process cold samples taken above, with
    # this process's hot numbers for the main config
    headline = {}
    if main_cold is not None:
        c, nopf, nopr = main_cold["cold"], main_cold.get("cold_no_prefault"), main_cold.get("cold_no_prime")
        pyc = main_cold["cold_python_process"]
        ms2 = lambda d: [round(d["median_us"] / 1e3, 3), round(d["p90_us"] / 1e3, 3)] if d else None  # noqa: E731
        headline[args.model] = headline_entry(
            c["median_us"] / 1e3, c["p90_us"] / 1e3, c["n"], hot_max, direct_max, main_cold["breakdown"],
            c["kernels_loaded"], main_cold["launches"],
            {"nopf_ms": ms2(nopf), "noprime_ms": ms2(nopr),
             "py_ms": ([round(pyc["median_us"] / 1e3, 3), round(pyc["p90_us"] / 1e3, 3), pyc["n"]]
                       if pyc else None)})
        for m, blk in configs_detail.items():
            c = blk["cold"]
            headline[m] = headline_entry(c["median_us"] / 1e3, c["p90_us"] / 1e3, c["n"],
                                         blk["hot_graph_us"] / 1e3, blk["hot_direct_us"] / 1e3,
                                         blk["breakdown"], c["kernels_loaded"], blk["launches"])

    phase("cpu baseline")
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        ts = time_oracle(spec, x, 5, 20.0)
        cpu = {"value": round(args.batch / statistics.mean(ts), 4), "unit": "imgs/s", "cores": cores_used(),
               "kind": "oracle", "cpu": cpu_model(),
               "sample": f"{len(ts)} full fp64 numpy-oracle forwards of a batch-{args.batch} {args.model} input"}

    st = cold_stats
    line = {
        "metric": METRIC,
        "value": round(world * args.batch * 1000.0 / hot_max, 2),
        "unit": "imgs/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(hot_max, 4),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "bf16",
        "data": "synthetic (seeded N(0,1) input, random-init weights of the architecture)",
        "config": {"workload": args.workload_name, "model": args.model,
                   "global_batch": world * args.batch, "per_gpu_batch": args.batch,
                   "parallelism": f"replicas{world}",
                   "packaging": ["one code object per kernel", "single code object",
                                 "operator families (memory-bound + contraction)",
                                 "cold start on a single function (both families behind one entry), "
                                 "repacked into the two family entries by pask_promote before the "
                                 "hot inferences"][args.packaging],
                   "branches": "independent nodes on a second stream" if args.branches else "one stream",
                   "hot_issue": "CUDA graph replay (captured on the 2nd inference)" if args.graph
                                else "direct cuLaunchKernelEx per layer",
                   "l2": "warm (no flush)" if args.no_flush else
                         "flushed (256 MiB memset) before every timed inference",
                   "cold": f"{args.cold_samples} fresh native processes per config (pask_cold), "
                           "t0 = pask_load_model entry, t1 = first inference done; an idle keeper "
                           "process holds a context meanwhile (GPU kept initialised)"},
        "e2e": {"value": round(world * args.batch * 1000.0 / e2e_max, 2), "unit": "imgs/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "ms_per_step": round(e2e_max, 4)},
        "gpu_launches": n_nodes * args.steps,
        "roofline": roofline,
        "cpu_baseline": cpu,
        "clocks": clocks,
        "wall_s_timed_region": round(w1 - w0, 4),
        "hot_ms": round(hot_max, 4),
        "hot_median_ms": round(hot_med_ms, 4),
        "hot_l2_warm_ms": round(warm_max, 4),
        "hot_direct_ms": round(direct_max, 4),
        "hot_direct_median_ms": round(hot_direct_med_ms, 4),
        "cold_inprocess_ms": round(cold_inproc_ms, 3),
        "kernels_loaded_names": loaded,
        "solutions_bound": solutions,
        "code_objects_loaded": st["code_objects_loaded"],
        "plan": {"queries": st["queries"], "hits": st["hits"], "lookups": st["lookups"],
                 "reused_nodes": sum(1 for b in plan if b[3] == 1)},
        "per_kernel_roofline": per_kernel_roofline,
        "cold_detail": main_cold,
        "configs_detail": configs_detail or None,
    }
    # the LAST keys of the line (the driver keeps the tail of stdout): the
    # replica block (N > 1) or the compact per-config cold / hot block (N = 1)
    if replicas:
        line["replicas"] = replicas
    if headline:
        line["headline"] = {"legend": {"cold_ms": "med,p90,n (native procs)", "hot_ms": "graph,direct",
                                       "cold/hot": "graph,direct", "util": "busy/cold",
                                       "bd_us": "/".join(BREAKDOWN_KEYS), "py_ms": "PyTorch procs"},
                            **headline}
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
