"""Cold-start samples in fresh processes (SURVEY.md §8(d) protocol).

Each sample is a new Python process: import torch, create the context, upload
weights, synchronise, pask_create (all outside the window), then
t0 = pask_load_model entry, t1 = first inference complete.  The parent prints
the median / p90 per scheme and the paper's breakdown (Fig. 1(b) / Fig. 7
analog: loading exposed / issue / GPU / other).

    python scripts/cold_samples.py --model resnet50 --n 20 [--schemes pask,pask_i,...]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# scheme -> pask_config keywords
SCHEMES = {
    "pask": dict(),                                   # default: caller uploads, helper encodes
    "pask_thread": dict(proactive=1),                 # async loader thread
    "pask_interleave": dict(proactive=1, interleave=1),  # Fig. 5 interleaving
    "pask_single_image": dict(packaging=1),           # whole catalog as one code object
    "pask_families": dict(packaging=2),               # operator families (D8)
    "pask_single_function": dict(packaging=3),        # both families in one CUfunction (D10)
    "pask_families_branches": dict(packaging=2, branches=1),  # bench default: + side stream (D9)
    "pask_families_branches_1s": dict(packaging=2, branches=1),  # ... cold issue on one stream
    "pask_families_branches_noevw": dict(packaging=2, branches=1),  # ... events not warmed at create
    "pask_i": dict(reuse=0),                          # PaSK-I: proactive, no reuse
    "pask_r": dict(search=1),                         # PaSK-R: naive (exhaustive-order) search
    "reactive": dict(proactive=0, reuse=0),           # Baseline analog: lazy load at first launch
    "reactive_reuse": dict(proactive=0),              # reuse without the proactive loader
    # tuned library (per-problem specialised conv solutions)
    "baseline_tuned": dict(catalog=1, proactive=0, reuse=0),  # the paper's Baseline
    "pask_tuned": dict(catalog=1),                    # PASK over the tuned library
    "pask_encfirst": dict(),                          # experiment: caller encodes, then uploads
}
SCHEME_ENV = {"pask_encfirst": {"PASK_ENCODE_FIRST": "1"},
              "pask_families_branches_1s": {"PASK_DIRECT_ONE_STREAM": "1"},
              "pask_families_branches_noevw": {"PASK_NO_EVENT_WARM": "1"}}


def child(model, scheme, batch=1):
    import torch

    from paper_conf_dac_huangdxz25_b200 import pask as P
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from workloads import build_model
    spec, x = build_model(model, **({"batch": batch} if batch != 1 else {}))
    dm = DeviceModel(spec)
    dm.set_input(x)
    torch.cuda.synchronize()
    ctx = P.Context(0, P.config(**SCHEMES[scheme]))
    s = torch.cuda.current_stream().cuda_stream
    time.sleep(float(os.environ.get("PASK_COLD_SLEEP_MS", "50")) / 1e3)  # idle before the cold window
    torch.cuda.synchronize()
    t0 = time.perf_counter_ns()
    ctx.load_model(dm.graph, plan=False)
    ctx.infer(s)
    ctx.sync()
    t1 = time.perf_counter_ns()
    st = ctx.stats()
    tl = {}
    for k in range(P.num_kernels()):
        ld, rd, lb = ctx.kernel_timeline(k)
        if ld:
            tl[P.kernel_name(k)[5:]] = [round(lb / 1e3), round(ld / 1e3), round(rd / 1e3)]
    # hot (L2-warm) for the ratio, same process
    for _ in range(10):
        ctx.infer(s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(50):
        ctx.infer(s)
    e1.record()
    torch.cuda.synchronize()
    st2 = ctx.stats()
    hot_issue = (st2["issue_ns"] - st["issue_ns"]) / 1e3 / max(1, st2["launches"] - st["launches"])
    print(json.dumps({"hot_issue_us_per_launch": hot_issue,
                      "cold_issue_us_per_launch": st["issue_ns"] / 1e3 / max(1, st["launches"]),
                      "cold_us": st["cold_wall_ns"] / 1e3, "cold_py_us": (t1 - t0) / 1e3, "hot_us": 1e3 * e0.elapsed_time(e1) / 50,
                      "kernels_loaded": st["kernels_loaded"], "code_objects": st["code_objects_loaded"],
                      "load_us": st["load_ns"] / 1e3, "load_exposed_us": st["load_exposed_ns"] / 1e3,
                      "issue_us": st["issue_ns"] / 1e3, "gpu_span_us": st["gpu_span_ns"] / 1e3,
                      "plan_us": st["plan_ns"] / 1e3, "encode_us": st["encode_ns"] / 1e3,
                      "t_load_done_us": st["load_done_ns"] / 1e3, "t_infer_entry_us": st["infer_entry_ns"] / 1e3,
                      "t_first_launch_us": st["first_launch_ns"] / 1e3,
                      "t_last_launch_us": st["last_launch_ns"] / 1e3,
                      "t_encode_begin_us": st["encode_begin_ns"] / 1e3,
                      "t_encode_end_us": st["encode_end_ns"] / 1e3,
                      "timeline": tl}))
    ctx.close()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="resnet50")
    ap.add_argument("--n", type=int, default=20)
    ap.add_argument("--schemes", default=",".join(SCHEMES))
    ap.add_argument("--child", default=None)
    ap.add_argument("--batch", type=int, default=1)
    a = ap.parse_args()
    if a.child:
        child(a.model, a.child, a.batch)
        return
    out = {}
    for scheme in a.schemes.split(","):
        samples = []
        for _ in range(a.n):
            r = subprocess.run([sys.executable, __file__, "--model", a.model, "--child", scheme,
                                "--batch", str(a.batch)],
                               capture_output=True, text=True, timeout=300,
                               env={**os.environ, **SCHEME_ENV.get(scheme, {})})
            line = [l for l in r.stdout.splitlines() if l.startswith("{")]
            if not line:
                print(r.stderr[-2000:], file=sys.stderr)
                continue
            samples.append(json.loads(line[-1]))
        if not samples:
            continue
        print(f"   {scheme} first-sample timeline [lib, load, ready_at] us: {samples[0]['timeline']}",
              flush=True)
        med = {k: statistics.median(s[k] for s in samples) for k in samples[0] if k != "timeline"}
        cold = sorted(s["cold_us"] for s in samples)
        med["cold_p90_us"] = cold[min(len(cold) - 1, int(0.9 * len(cold)))]
        med["cold_over_hot"] = med["cold_us"] / med["hot_us"]
        med["n"] = len(samples)
        out[scheme] = med
        print(f"{a.model:12s} {scheme:18s} cold med {med['cold_us']:8.1f} p90 {med['cold_p90_us']:8.1f} us"
              f"  hot {med['hot_us']:7.1f}  ratio {med['cold_over_hot']:5.2f}  kernels {med['kernels_loaded']:.0f}"
              f"  load {med['load_us']:6.1f} exposed {med['load_exposed_us']:6.1f} issue {med['issue_us']:6.1f}"
              f" gpu {med['gpu_span_us']:6.1f} issue/launch cold {med['cold_issue_us_per_launch']:4.2f}"
              f" hot {med['hot_issue_us_per_launch']:4.2f} | t: loads {med['t_load_done_us']:6.1f} infer {med['t_infer_entry_us']:6.1f}"
              f" first {med['t_first_launch_us']:6.1f} last {med['t_last_launch_us']:6.1f}"
              f" encode [{med['t_encode_begin_us']:6.1f}, {med['t_encode_end_us']:6.1f}]", flush=True)
    print(json.dumps({"model": a.model, "schemes": out}))


if __name__ == "__main__":
    main()
