"""bench.py -- GMP-SVM hot path on B200: train + predict on the MNIST-shaped workload.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gmpsvm|reference] [--eps E]
    torchrun --nproc-per-node N bench.py --gpus N ...      (pairs / test rows sharded, NCCL gathers)

One step = one whole pass of the hot path on the workload
BASELINE.json's metric is quoted on (configs[2]: MNIST-shaped 60k train / 10k test x 784,
10 classes, gamma 0.125, C 10): gmpsvm_train + gmpsvm_predict_proba.  Inputs are resident
in HBM when the timed region starts (`value`); `e2e` repeats the step through the C ABI
from pinned host buffers with the H2D/D2H copies inside the timed region.

Prints ONE JSON line on rank 0.  The metric is time-like (seconds per train+predict job),
so higher_is_better = false.
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import shutil
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# the solver runs pair groups on concurrent streams: give them distinct hardware queues
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import datagen  # noqa: E402

METRIC = "train+predict sec on MNIST-shaped 60k×784×10; kernel GFLOP/s vs peak"
FP32_PEAK_TFLOPS_DERIVED = 148 * 128 * 2 * 1.965e9 / 1e12  # SMs x FP32 lanes x 2 x max SM clock


def _fp32_peak():
    """Measured FFMA peak (tools/micro/ffma_peak.cu, profiles/fp32_ffma_peak.json), else derived."""
    try:
        return float(json.load(open(os.path.join(ROOT, "profiles", "fp32_ffma_peak.json")))["sustained_tflops"])
    except Exception:
        return FP32_PEAK_TFLOPS_DERIVED


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region (B200_PROFILING.md)."""

    # no power.draw: reading it holds the driver long enough to stall a concurrent step's host
    # calls (30 ms outlier steps were seen with it in the query)
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._th = None

    def sample(self):
        try:
            out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                  "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5)
            f = [x.strip() for x in out.stdout.strip().split(",")]
            if len(f) >= 6:
                self.samples.append(f)
        except Exception:
            pass

    def _run(self):
        if os.environ.get("GMPSVM_BENCH_CLOCKS") == "off":  # diagnostics only: no sampler process
            return
        # one long-running nvidia-smi (the recipe's `-lms 200` loop): NVML is initialised once, so
        # the sampling does not stall the host's CUDA calls the way a fresh process every 0.2 s did
        try:
            lb = ["stdbuf", "-oL"] if shutil.which("stdbuf") else []  # a line per sample through the pipe
            self._proc = subprocess.Popen([*lb, "nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                           "--format=csv,noheader,nounits", "-lms", "200"],
                                          stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self._proc = None
            return
        for line in self._proc.stdout:
            f = [x.strip() for x in line.strip().split(",")]
            if len(f) >= 6:
                self.samples.append(f)
            if self._stop.is_set():
                break

    def __enter__(self):
        self._proc = None
        self._th = threading.Thread(target=self._run, daemon=True)
        self._th.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._proc is not None:
            self._proc.terminate()
            try:
                self._proc.wait(timeout=5)
            except Exception:
                self._proc.kill()
        if self._th:
            self._th.join(timeout=10)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[2 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def _env_dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def lpt_shards(sizes, n_shards):
    """Longest-processing-time-first assignment of pairs (cost ~ n_p^1.5) to ranks."""
    order = np.argsort(-np.asarray(sizes, dtype=np.float64) ** 1.5, kind="stable")
    load = np.zeros(n_shards)
    out = [[] for _ in range(n_shards)]
    for p in order:
        r = int(np.argmin(load))
        out[r].append(int(p))
        load[r] += float(sizes[p]) ** 1.5
    return [sorted(o) for o in out]


# ------------------------------------------------------------------------------------------ oracle arms
def cpu_sample(spec, eps, n_train=6000, n_test=1000):
    """The oracle, as it stands, on a bounded sample of the same workload (host cores)."""
    import oracle

    _, X, y, Xt, yt = datagen.make_config(spec.name, n_train=n_train, n_test=n_test)
    t0 = time.perf_counter()
    m = oracle.train(X, y, spec.k, spec.C, spec.gamma, eps)
    t1 = time.perf_counter()
    oracle.predict(m, X, y, Xt, want_dec=False)
    t2 = time.perf_counter()
    return t2 - t0, t1 - t0, t2 - t1, oracle.default_threads()


def run_reference(args, spec):
    ws, rank, _ = _env_dist()
    if rank != 0:
        return 0
    for _ in range(args.warmup):
        cpu_sample(spec, args.eps)
    times = []
    for _ in range(args.steps):
        t, tt, tp, cores = cpu_sample(spec, args.eps)
        times.append(t)
    v = float(np.mean(times))
    sample = (f"oracle (FP64 C++ WSS2 SMO + LLW sigmoid + exact WLW coupling) on a 10% sample of the workload: "
              f"6000 train / 1000 test MNIST-shaped rows, eps={args.eps:g}, {cores} host threads")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "s (sample)", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": v * 1e3, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": _config(spec, args),
            "cpu_baseline": {"value": v, "unit": "s (sample)", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": "s (sample)", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def _config(spec, args):
    return {"workload": f"{spec.name}-shaped {spec.n_train} train / {spec.n_test} test x {spec.d}, k={spec.k}, "
                        f"C={spec.C:g}, gamma={spec.gamma:g}, eps={args.eps:g}",
            "n_train": spec.n_train, "n_test": spec.n_test, "d": spec.d, "k": spec.k, "C": spec.C,
            "gamma": spec.gamma, "eps": args.eps, "ws_size": args.ws_size, "q": args.q or args.ws_size // 2,
            "parallelism": f"pairs+test-rows x{args.gpus}",
            "l2": "inputs larger than L2 (X 188 MB, kernel matrix 14.4 GB > 126 MB L2); no flush needed"}


# ------------------------------------------------------------------------------------------ GPU arm
def run_gpu(args, spec):
    import torch
    import torch.distributed as dist

    import paper_conf_icde_wenshcc19_b200 as gm
    from paper_conf_icde_wenshcc19_b200 import dist as gdist

    ws, rank, local = _env_dist()
    # one rank per GPU; GMPSVM_DIST_BACKEND=gloo with more ranks than GPUs is a plumbing check only
    gpu = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if ws > 1:
        backend = os.environ.get("GMPSVM_DIST_BACKEND", "nccl")
        dist.init_process_group(backend, device_id=dev if backend == "nccl" else None)
    _, X, y, Xt, yt = datagen.make_config(spec.name)
    Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
    Xp, yp, Xtp = (torch.from_numpy(X).pin_memory(), torch.from_numpy(y).pin_memory(),
                   torch.from_numpy(Xt).pin_memory())
    stream = torch.cuda.current_stream(dev)
    opts = dict(ws_size=args.ws_size, q=args.q)
    if args.inner_cap:
        opts["inner_iter_cap"] = args.inner_cap

    host_ms = []  # host-clock duration of each step's calls (diagnostic: stalls outside the GPU)

    def step(Xa, ya, Xta, host=False):
        t0 = time.perf_counter()
        if ws > 1:
            model, prob = gdist.train_predict(Xa, ya, Xta, spec.k, spec.C, spec.gamma, args.eps, **opts)
        else:
            model = gm.train(Xa, ya, spec.k, spec.C, spec.gamma, args.eps, **opts)
            t1 = time.perf_counter()
            prob = model.predict_proba(Xta)
            host_ms.append((round((t1 - t0) * 1e3, 2), round((time.perf_counter() - t1) * 1e3, 2)))
        return model, prob

    # the clock sampler (an nvidia-smi process every 0.2 s) starts during the warm-up, so its
    # start-up cost does not land in the first timed step
    clk = ClockSampler(gpu).__enter__()
    t_wait = time.time()  # first sample before the warm-up: the GPU must not idle between warm-up and timing
    while not clk.samples and clk._th.is_alive() and time.time() - t_wait < 10:
        time.sleep(0.05)
    gc.collect()
    gc.disable()  # no Python collector pauses from here through the e2e timed region
    for _ in range(args.warmup):
        model, prob = step(Xd, yd, Xtd)
    torch.cuda.synchronize(dev)
    n_warm = len(clk.samples)

    # ---- device-resident timed region
    t_ms, stats, pstats, nsvs = [], [], [], []
    try:
        l0 = gm.launch_count()
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        marks = []
        for _ in range(args.steps):
            model, prob = step(Xd, yd, Xtd)
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(stream)
            marks.append(ev)
            stats.append(getattr(model, "part_stats", None) or model.train_stats())
            pstats.append(gm.last_predict_stats())
            nsvs.append(model.n_sv)
        e1.record(stream)
        if len(clk.samples) <= n_warm:  # short timed region: one sample while its last step still runs
            clk.sample()
        torch.cuda.synchronize(dev)
        if ws > 1:
            dist.barrier()
        launches = gm.launch_count() - l0
    finally:
        clk.__exit__(None, None, None)
        del clk.samples[:n_warm]  # only samples taken during the timed region
    total_ms = e0.elapsed_time(e1)
    step_ms = [e0.elapsed_time(marks[0])] + [marks[i - 1].elapsed_time(marks[i]) for i in range(1, len(marks))]
    if ws > 1:
        t = torch.tensor([total_ms], device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms = total_ms / args.steps
    # the timed steps' output is checked, not just timed: every step's model has the same SV count
    # (deterministic kernels), the probabilities are finite rows summing to 1 (Eq 14) and classify
    # the test rows as the parity-tested model does (98.2 % on this workload; >= 97 % required)
    prob_np = prob.cpu().numpy() if hasattr(prob, "cpu") else np.asarray(prob)
    checks = {"n_sv_steps": sorted(set(nsvs)), "prob_finite": bool(np.isfinite(prob_np).all()),
              "prob_rowsum_maxdev": float(np.abs(prob_np.sum(1) - 1.0).max()),
              "test_accuracy": float((prob_np.argmax(1) == yt).mean()),
              "dec_path": int(pstats[-1].get("dec_path", -1))}
    if not (len(checks["n_sv_steps"]) == 1 and checks["prob_finite"] and checks["prob_rowsum_maxdev"] < 1e-9
            and checks["test_accuracy"] >= 0.97):
        raise SystemExit(f"bench: timed-step output check failed: {checks}")

    # ---- end to end from pinned host buffers (copies inside the timed region)
    Xh, yh, Xth = Xp.numpy(), yp.numpy(), Xtp.numpy()
    for _ in range(args.warmup):  # the host path runs on the library's own stream: warm its pool too
        model_h, prob_h = step(Xh, yh, Xth, host=True)
    torch.cuda.synchronize(dev)
    if ws > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        model_h, prob_h = step(Xh, yh, Xth, host=True)
    torch.cuda.synchronize(dev)
    e2e_ms = (time.perf_counter() - t0) * 1e3 / args.steps
    gc.enable()
    e2e_train = model_h.train_stats() if ws == 1 else getattr(model_h, "part_stats", {})
    e2e_pred = gm.last_predict_stats()
    if ws > 1:
        t = torch.tensor([e2e_ms], device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())

    if rank == 0:
        s = stats[-1]
        ps = pstats[-1]
        krow_ms = float(np.mean([x["t_kernel_ms"] for x in stats]))
        achieved = s["kernel_flops"] / (krow_ms * 1e-3) / 1e12
        peaks = _peaks()
        bf16 = peaks.get("bf16_tflops", 1590.0)
        # krow_contract runs on tcgen05 with a two-part (hi + lo) split and 3 MMAs per FP32-accurate
        # product (hi*hi + hi*lo + lo*hi): its speed of light is the dense peak of the MMA kind / 3.
        # Default kind::f16 (FP16 parts) at the measured bf16 burst peak (same dense rate for f16);
        # GMPSVM_SPLIT=tf32 uses kind::tf32 at bf16 x 0.5 (the guide's nominal 1.13 : 2.25 ratio)
        split = "tf32" if os.environ.get("GMPSVM_SPLIT", "") == "tf32" else "f16"
        mma_peak = bf16 * (0.5 if split == "tf32" else 1.0)
        peak = mma_peak / 3.0
        # lead mode: the contraction's main wave runs on all but the reserved SMs (the hardest pair's
        # solver holds those); frac_of_launch_sms scales the peak to the SMs the launch was given
        n_sms = torch.cuda.get_device_properties(dev).multi_processor_count
        lead_on = os.environ.get("GMPSVM_LEAD", "1") != "0"
        launch_sms = n_sms - (int(os.environ.get("GMPSVM_LEAD_RESERVE", "8")) if lead_on else 0)
        traffic = None
        tr_path = os.path.join(ROOT, "profiles", "krow_traffic.json")
        if os.path.exists(tr_path):
            traffic = json.load(open(tr_path)).get("dram_bytes_per_launch")
        line = {
            "metric": METRIC, "value": ms / 1e3, "unit": "s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (datagen mnist recipe, seeds 1234/1/2)",
            "config": _config(spec, args),
            "roofline": {"kernel": f"krow_contract (krow_tc_kernel, tcgen05 kind::{split}, 3-MMA hi/lo split)",
                         "bound": "tensor",
                         "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                         "traffic": traffic,
                         "peak_note": (f"kind::{split} dense = measured bf16 burst {bf16}"
                                       f"{' x 0.5' if split == 'tf32' else ''} = {mma_peak:.1f} TFLOP/s"
                                       f"{'' if 'bf16_tflops' in peaks else ' (fallback)'}; the hi/lo split needs 3 MMAs "
                                       "per FP32-accurate product, so peak = that / 3"),
                         "frac_of_launch_sms": achieved / (peak * launch_sms / n_sms),
                         "launch_sms": launch_sms,
                         "frac_of_mma_peak": achieved / mma_peak,
                         "frac_of_fp32_simt_peak": achieved / _fp32_peak(),
                         "fp32_simt_peak": _fp32_peak(),
                         "flops_per_launch": s["kernel_flops"], "launch_ms": krow_ms,
                         "algorithmic": "n(n+1)/2 kernel values x (2d+3) flop",
                         "schedule": ("lead mode (engine.cu): launch_ms spans the contraction's two launches, wave 0 "
                                      "(the hardest pair's class blocks) on every SM and wave 1 on 140 of 148 SMs while "
                                      "that pair's solver runs on the rest; GMPSVM_LEAD=0 times it alone"
                                      if os.environ.get("GMPSVM_LEAD", "1") != "0" else "alone (GMPSVM_LEAD=0)")},
            "phases_ms": {"stage": s["t_stage_ms"], "kernel_values": s["t_kernel_ms"], "select": s["t_select_ms"],
                          "subproblem": s["t_subproblem_ms"], "f_update": s["t_fupdate_ms"],
                          "finalize": s["t_finalize_ms"], "train_total": s["t_total_ms"],
                          "predict_stage": ps["t_stage_ms"], "decision_values": ps["t_decision_ms"],
                          "couple": ps["t_couple_ms"], "predict_total": ps["t_total_ms"]},
            "step_ms": step_ms,
            "host_ms_train_predict": host_ms[args.warmup:args.warmup + args.steps],
            "counters": {"outer_iters_max": s["outer_iters_max"], "inner_iters_sum": s["inner_iters_sum"],
                         "smo_cycles_per_step": s["smo_cycles_sum"] / max(1, s["inner_iters_sum"]),
                         "n_sv": s["n_sv"], "dec_tflops": ps["dec_flops"] / (ps["t_decision_ms"] * 1e-3) / 1e12
                         if ps["t_decision_ms"] > 0 else None},
            "checks": checks,
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "e2e": {"value": e2e_ms / 1e3, "unit": "s", "h2d_bytes_per_step": int(X.nbytes + y.nbytes + Xt.nbytes),
                    "d2h_bytes_per_step": int(prob_h.nbytes),
                    "train_total_ms": e2e_train.get("t_total_ms"), "train_stage_ms": e2e_train.get("t_stage_ms"),
                    "predict_total_ms": e2e_pred["t_total_ms"], "predict_stage_ms": e2e_pred["t_stage_ms"]},
        }
        # the int8-digit decision-value contraction (dec_i8.cu): executed int8 tensor-core work =
        # 19 digit products x 2 d ops per (test row, SV); peak = int8 dense = 2 x the measured bf16
        if ps.get("dec_path", -1) == 1 and ps["t_decision_ms"] > 0:
            i8_ops = X.shape[1] * 2.0 * 19 * Xt.shape[0] * s["n_sv"]
            i8_peak = 2.0 * bf16
            line["dec_roofline"] = {"kernel": "dec_i8_kernel (tcgen05 kind::i8, 5 int8 digit planes, 19 products)",
                                    "bound": "tensor", "achieved": i8_ops / (ps["t_decision_ms"] * 1e-3) / 1e12,
                                    "peak": i8_peak, "unit": "TOP/s (int8)",
                                    "frac": i8_ops / (ps["t_decision_ms"] * 1e-3) / 1e12 / i8_peak,
                                    "decision_ms": ps["t_decision_ms"],
                                    "algorithmic_tflops": ps["dec_flops"] / (ps["t_decision_ms"] * 1e-3) / 1e12}
        if not args.no_cpu_baseline and ws == 1:
            v, tt, tp, cores = cpu_sample(spec, args.eps)
            line["cpu_baseline"] = {"value": v, "unit": "s (sample)", "cores": cores, "kind": "oracle",
                                    "sample": f"6000 train / 1000 test MNIST-shaped rows (10% of the workload), "
                                              f"eps={args.eps:g}: train {tt:.1f} s + predict {tp:.1f} s"}
        full_ref = os.path.join(ROOT, "profiles", "r02", "cpu_full_mnist_r02.json")
        if os.path.exists(full_ref) and spec.name == "mnist":
            # the oracle once on the FULL workload on a GPU box's host (tools/cpu_full.py, committed:
            # ~2 minutes on 16 threads, too long to repeat in every bench run)
            fr = json.load(open(full_ref))
            line["cpu_baseline_full"] = {"value": fr["total_s"], "unit": "s", "train_s": fr["train_s"],
                                         "predict_s": fr["predict_s"], "cores": fr["threads"],
                                         "cpu_model": fr["cpu_model"], "kind": "oracle",
                                         "source": "profiles/r02/cpu_full_mnist_r02.json (tools/cpu_full.py)"}
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gmpsvm", choices=["gmpsvm", "reference"])
    ap.add_argument("--config", default="mnist")
    ap.add_argument("--eps", type=float, default=1e-3)
    ap.add_argument("--ws-size", dest="ws_size", type=int, default=192)
    ap.add_argument("--q", type=int, default=0, help="new working-set rows per outer iteration (0: ws_size / 2)")
    ap.add_argument("--inner-cap", dest="inner_cap", type=int, default=0, help="local SMO steps per outer iteration cap (0: 100 ws_size)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    spec = datagen.CONFIGS[args.config]
    if args.impl == "reference":
        return run_reference(args, spec)
    return run_gpu(args, spec)


if __name__ == "__main__":
    sys.exit(main())
