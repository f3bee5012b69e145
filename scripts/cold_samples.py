"""Cold-start samples in fresh native processes (SURVEY.md §8(d) protocol).

Each sample is a new process of the native sampler
(paper_conf_dac_huangdxz25_b200/pask_cold, csrc/tools/pask_cold.cpp): it
creates the context, uploads the weights and the input, synchronises and calls
pask_create, all outside the window; then t0 = pask_load_model entry and t1 =
the first inference complete (the library's cold_wall_ns).  The parent writes
the lowered model once as a model image (DeviceModel.save_image) and runs the
children; no child imports Python or PyTorch, so a sample costs ~0.1-0.5 s.

    python scripts/cold_samples.py --model resnet50 --n 20 [--schemes pask,pask_i,...]

Also the replica harness of SURVEY.md §8(e): N children cold-starting
together (each prints "ready" and waits for a line on stdin; the parent
releases them at once), on one GPU (--replicas) or one per GPU.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
EXE = os.path.join(ROOT, "paper_conf_dac_huangdxz25_b200", "pask_cold")

# scheme -> pask_config fields
SCHEMES = {
    "pask": dict(),                                      # library default: caller uploads, helper encodes
    "pask_thread": dict(proactive=1),                    # async loader thread
    "pask_interleave": dict(proactive=1, interleave=1),  # Fig. 5 interleaving
    "pask_single_image": dict(packaging=1),              # whole catalog as one code object
    "pask_families": dict(packaging=2),                  # operator families (D8)
    "pask_single_function": dict(packaging=3),           # both families in one CUfunction (D10)
    "pask_families_branches": dict(packaging=2, branches=1),  # bench default: + side stream (D9)
    "pask_i": dict(reuse=0),                             # PaSK-I: proactive, no reuse
    "pask_r": dict(search=1),                            # PaSK-R: naive (exhaustive-order) search
    "reactive": dict(proactive=0, reuse=0),              # Baseline analog: lazy load at first launch
    "reactive_reuse": dict(proactive=0),                 # reuse without the proactive loader
    # tuned library (per-problem specialised conv solutions)
    "baseline_tuned": dict(catalog=1, proactive=0, reuse=0),  # the paper's Baseline
    "pask_tuned": dict(catalog=1),                       # PASK over the tuned library
}


def cfg_arg(cfg: dict) -> str:
    return ",".join(f"{k}={int(v)}" for k, v in sorted(cfg.items())) or "reuse=1"


def write_image(model: str, path: str | None = None, batch: int = 1) -> str:
    """The lowered model + weights + seeded input as a model image (host only)."""
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from workloads import build_model
    spec, x = build_model(model, **({"batch": batch} if batch != 1 else {}))
    if path is None:
        path = os.path.join(tempfile.gettempdir(), f"pask_{model}_b{batch}_{os.getpid()}.pmodel")
    DeviceModel(spec, alloc=False).save_image(path, x)
    return path


def run_child(image: str, cfg: dict, device: int = 0, hot: int = 0, dump: str | None = None,
              flush_mb: int = 256, timeout: float = 120.0, env: dict | None = None,
              promote: bool | None = None) -> dict:
    """One fresh native process.  promote (default: with hot inferences under
    packaging 3) calls pask_promote after the cold inference -- the idle-interval
    repack into the two family entries (D15) -- before the hot ones."""
    cmd = [EXE, image, "--cfg", cfg_arg(cfg), "--device", str(device)]
    if promote is None:
        promote = bool(hot) and cfg.get("packaging") == 3
    if promote:
        cmd += ["--promote"]
    if hot:
        cmd += ["--hot", str(hot), "--flush-mb", str(flush_mb)]
    if dump:
        cmd += ["--dump", dump]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout,
                       env={**os.environ, **(env or {})})
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    if r.returncode != 0 or not lines:
        raise RuntimeError(f"pask_cold failed (rc {r.returncode}): {r.stderr[-2000:]}")
    return json.loads(lines[-1])


def py_child(model: str, cfg: dict, batch: int = 1):
    """A cold start in a fresh PyTorch process (the framework process a model
    server runs in): torch allocates and uploads, pask_create, 50 ms idle, then
    the cold window.  Prints the same keys as the native sampler."""
    import time

    import torch

    from paper_conf_dac_huangdxz25_b200 import pask as P
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from workloads import build_model
    spec, x = build_model(model, **({"batch": batch} if batch != 1 else {}))
    dm = DeviceModel(spec)
    dm.set_input(x)
    torch.cuda.synchronize()
    ctx = P.Context(0, P.config(**cfg))
    s = torch.cuda.current_stream().cuda_stream
    time.sleep(0.05)
    torch.cuda.synchronize()
    ctx.load_model(dm.graph, plan=False)
    ctx.infer(s)
    ctx.sync()
    st = ctx.stats()
    print(json.dumps({"cold_us": st["cold_wall_ns"] / 1e3, "kernels_loaded": st["kernels_loaded"],
                      "t_load_done_us": st["load_done_ns"] / 1e3, "gpu_span_us": st["gpu_span_ns"] / 1e3}))
    ctx.close()


def run_py_child(model: str, cfg: dict, batch: int = 1, timeout: float = 300.0) -> dict:
    r = subprocess.run([sys.executable, os.path.abspath(__file__), "--py-child", model, "--cfg", cfg_arg(cfg),
                        "--batch", str(batch)], capture_output=True, text=True, timeout=timeout)
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    if r.returncode != 0 or not lines:
        raise RuntimeError(f"python cold child failed (rc {r.returncode}): {r.stderr[-2000:]}")
    return json.loads(lines[-1])


def pctl(vals, q):
    s = sorted(vals)
    return s[min(len(s) - 1, int(q * len(s)))]


def sample(image: str, cfg: dict, n: int, device: int = 0) -> list[dict]:
    return [run_child(image, cfg, device) for _ in range(n)]


class Keeper:
    """An idle process holding a CUDA context on `device` while fresh-process
    samples run (a pask_cold child set up and blocked before its cold window):
    the GPU stays initialised between children, as under a persistence daemon,
    instead of being torn down and re-initialised for each (~1 s per child).
    Measured on one box (profiles/r2/r3h_keeper.log, 12 children per row): the
    children's cold medians with and without it are within the box noise."""

    def __init__(self, image: str, cfg: dict, device: int = 0):
        self.cmd = [EXE, image, "--cfg", cfg_arg(cfg), "--device", str(device), "--wait"]
        self.proc = None

    def __enter__(self):
        self.proc = subprocess.Popen(self.cmd, stdin=subprocess.PIPE, stdout=subprocess.PIPE,
                                     stderr=subprocess.PIPE, text=True)
        line = self.proc.stdout.readline()
        if line.strip() != "ready":
            self.proc.kill()
            self.proc.wait()
            raise RuntimeError(f"keeper did not get ready: {line!r} {self.proc.stderr.read()[-2000:]}")
        return self

    def __exit__(self, *exc):
        self.proc.kill()            # our own child, by PID; it never entered its cold window
        self.proc.wait()
        return False


def summarize(samples: list[dict]) -> dict:
    cold = [s["cold_us"] for s in samples]
    return {"median_us": statistics.median(cold), "p90_us": pctl(cold, 0.9), "min_us": min(cold),
            "n": len(cold), "kernels_loaded": samples[0]["kernels_loaded"]}


def breakdown(samples: list[dict]) -> dict:
    """Partition of the cold wall (Fig. 1(b) / Fig. 7 categories, reading G1:
    loading / issue / GPU execution / other) from timeline = 1 samples, per
    sample then median:
      plan       pask_load_model entry -> plan done (parse + Algorithm 1)
      load       plan done -> every planned kernel uploaded (encode overlaps it)
      issue      uploads done -> first launch issued (infer entry, first launch)
      gpu_busy   union of the kernels' [start, end] intervals (timeline stamps)
      gpu_idle   first launch -> end of the event span, minus busy (issue-paced
                 gaps; for schemes that load during the issue, the GPU waiting
                 for those loads)
      other      the rest of the window (sync return)
    The six parts sum to the cold wall.
    and GPU utilisation = gpu_busy / cold wall (Fig. 6(b))."""
    rows = []
    for s in samples:
        cold = s["cold_us"]
        plan = s["plan_us"]
        first = s["t_first_launch_us"]
        # schemes that load during the issue (reactive, loader thread, interleave):
        # loads after the first launch show up as GPU idle (the GPU waits for them)
        ld = min(s["t_load_done_us"], first)
        load = max(0.0, ld - plan)
        issue = max(0.0, first - max(plan, ld))
        window = cold - first                              # first launch -> t1
        busy = min(s["gpu_busy_us"], window)
        other = max(0.0, window - s["gpu_span_us"])        # outside the event span: the sync return
        idle = max(0.0, window - busy - other)
        rows.append({"plan": plan, "load": load, "issue": issue, "gpu_busy": busy, "gpu_idle": idle,
                     "other": other, "cold": cold, "util": busy / cold if cold else 0.0})
    return {k: round(statistics.median(r[k] for r in rows), 1 if k != "util" else 4) for k in rows[0]}


def replicas(image: str, cfg: dict, n_procs: int, trials: int, devices=None, dump_dir: str | None = None,
             timeout: float = 120.0) -> list[list[dict]]:
    """trials x n_procs cold starts; in each trial the n_procs children are
    released into the cold window together (devices[i] per child, default all
    on device 0: loader contention on one GPU's driver and host)."""
    devices = devices or [0] * n_procs
    out = []
    for t in range(trials):
        procs = []
        for i in range(n_procs):
            cmd = [EXE, image, "--cfg", cfg_arg(cfg), "--device", str(devices[i]), "--wait"]
            if dump_dir and t == 0:
                cmd += ["--dump", os.path.join(dump_dir, f"replica{i}.bin")]
            procs.append(subprocess.Popen(cmd, stdin=subprocess.PIPE, stdout=subprocess.PIPE,
                                          stderr=subprocess.PIPE, text=True))
        for p in procs:  # every child set up and waiting
            line = p.stdout.readline()
            if line.strip() != "ready":
                raise RuntimeError(f"replica did not get ready: {line!r} {p.stderr.read()[-2000:]}")
        for p in procs:  # release them together
            p.stdin.write("go\n")
            p.stdin.flush()
        res = []
        for p in procs:
            so, se = p.communicate(timeout=timeout)
            lines = [l for l in so.splitlines() if l.startswith("{")]
            if p.returncode != 0 or not lines:
                raise RuntimeError(f"replica failed (rc {p.returncode}): {se[-2000:]}")
            res.append(json.loads(lines[-1]))
        out.append(res)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="resnet50")
    ap.add_argument("--n", type=int, default=20)
    ap.add_argument("--schemes", default=",".join(SCHEMES))
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--hot", type=int, default=200, help="hot inferences of one extra child per scheme")
    ap.add_argument("--replicas", default=None,
                    help="e.g. 1,2,4,8: N processes on ONE GPU released into the cold start together "
                         "(SURVEY.md §8(e) loader contention), --n trials each")
    ap.add_argument("--py-child", default=None, help=argparse.SUPPRESS)
    ap.add_argument("--cfg", default="", help=argparse.SUPPRESS)
    a = ap.parse_args()
    if a.py_child:
        py_child(a.py_child, {k: int(v) for k, v in (kv.split("=") for kv in a.cfg.split(",") if kv)}, a.batch)
        return
    image = write_image(a.model, batch=a.batch)
    if a.replicas:
        cfg = SCHEMES["pask_families_branches"]
        res = {}
        try:
            for n in [int(v) for v in a.replicas.split(",")]:
                trials = replicas(image, cfg, n, a.n)
                cold = [r["cold_us"] for t in trials for r in t]
                per = [[round(t[i]["cold_us"], 1) for t in trials] for i in range(n)]
                res[n] = {"cold_med_us": statistics.median(cold), "cold_p90_us": pctl(cold, 0.9),
                          "cold_max_us": max(cold), "trials": a.n,
                          "per_replica_med_us": [round(statistics.median(v), 1) for v in per],
                          "kernels_loaded": sorted({int(r["kernels_loaded"]) for t in trials for r in t}),
                          "load_done_med_us": statistics.median(r["t_load_done_us"] for t in trials for r in t)}
                base = res[min(res)]["cold_med_us"]
                res[n]["contention"] = res[n]["cold_med_us"] / base
                print(f"{a.model} replicas {n}: cold med {res[n]['cold_med_us']:7.1f} p90 {res[n]['cold_p90_us']:7.1f} "
                      f"max {res[n]['cold_max_us']:7.1f} us  contention {res[n]['contention']:.2f}  load_done "
                      f"{res[n]['load_done_med_us']:6.1f}  kernels {res[n]['kernels_loaded']}  per-replica "
                      f"{res[n]['per_replica_med_us']}", flush=True)
        finally:
            os.unlink(image)
        print(json.dumps({"model": a.model, "replicas_one_gpu": res}))
        return
    out = {}
    try:
        for scheme in a.schemes.split(","):
            cfg = SCHEMES[scheme]
            samples = sample(image, cfg, a.n)
            tl = sample(image, {**cfg, "timeline": 1}, max(5, a.n // 2))
            hot = run_child(image, cfg, hot=a.hot) if a.hot else None
            med = summarize(samples)
            med["breakdown_us"] = breakdown(tl)
            med["hot_direct_us"] = hot["hot_median_us"] if hot else None
            med["cold_over_hot_direct"] = med["median_us"] / hot["hot_median_us"] if hot else None
            med["queries"], med["hits"], med["lookups"] = (samples[0]["queries"], samples[0]["hits"],
                                                          samples[0]["lookups"])
            med["timeline"] = samples[0]["timeline"]
            out[scheme] = med
            bd = med["breakdown_us"]
            print(f"{a.model:12s} {scheme:22s} cold med {med['median_us']:8.1f} p90 {med['p90_us']:8.1f} us"
                  f" (n {med['n']})  hot(direct) {med['hot_direct_us'] or 0:7.1f}  ratio "
                  f"{med['cold_over_hot_direct'] or 0:5.2f}  kernels {med['kernels_loaded']:.0f}  "
                  f"q/h/l {med['queries']:.0f}/{med['hits']:.0f}/{med['lookups']:.0f} | plan {bd['plan']} "
                  f"load {bd['load']} issue {bd['issue']} busy {bd['gpu_busy']} idle {bd['gpu_idle']} "
                  f"other {bd['other']} util {bd['util']}", flush=True)
    finally:
        os.unlink(image)
    print(json.dumps({"model": a.model, "batch": a.batch, "schemes": out}))


if __name__ == "__main__":
    main()
