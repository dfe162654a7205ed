#!/usr/bin/env python
"""Benchmark of the B200 Hilbert-BVH Barnes-Hut step (BASELINE.json metric:
"BH step time & bodies/s (theta=0.5, N=10M) at 1/2/4/8 B200; interactions/s").

Workload: config 3 of BASELINE.json -- two-disk galaxy collision, N = 10^7,
theta = 0.5, eps = 1e-3, dt = 1e-3, fixed 16-bit Hilbert grid (DESIGN.md
A8), synthetic seeded input (workloads/).  A "step" is one full pass of
Alg. 6: bbox, keys, radix sort, permute, build, force, leapfrog.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Prints one JSON line (rank 0).  For N > 1 launch with torch.distributed.run.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workloads import CONFIGS, generate  # noqa: E402

FLOPS_PER_INTERACTION = 20  # 3 sub + 3 mul/fma (r^2) + eps add + rsqrt + 3 mul + 3 fma ~ 20 flop
UNIT = "bodies/s"


def n_str(n: int) -> str:
    for div, suf in ((10 ** 9, "G"), (10 ** 6, "M"), (10 ** 3, "k")):
        if n % div == 0:
            return f"{n // div}{suf}"
    return str(n)


def metric_name(cfg) -> str:
    """BASELINE.json's metric for the workload actually run."""
    return f"BH step bodies/s (theta={cfg['theta']:g}, N={n_str(cfg['n'])})"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="cfg3")
    ap.add_argument("--n", type=int, default=0, help="override N (testing only)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target oracle force-sample time")
    ap.add_argument("--exchange", choices=["peer", "nccl"], default="peer",
                    help="multi-GPU exchange: fused update + peer-memory stores (default) or NCCL all-gather")
    ap.add_argument("--balance", choices=["cost", "equal"], default="cost",
                    help="multi-GPU ranges (peer exchange): cost-weighted from the last pass (NEXT-3(i), default) "
                         "or equal slices [A21]")
    ap.add_argument("--precision", type=int, choices=[32, 64], default=32,
                    help="32: fp32 state and interactions (default); 64: the paper's FP64 throughout (NEXT-2)")
    ap.add_argument("--sort-every", type=int, default=1,
                    help="ablation: tree reuse, re-sort every k-th step (NEXT-3(iii)); 1 = Alg. 6")
    ap.add_argument("--repeats", type=int, default=5, help="timed repeats of K steps (median reported, SURVEY 8(d))")
    ap.add_argument("--key-bits", type=int, default=16, help="Hilbert grid bits per axis (0 = paper count rule)")
    ap.add_argument("--no-extras", action="store_true",
                    help="skip the extra blocks of the default run (FP64 mode, config 2, all-pairs calibration)")
    return ap.parse_args()


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def workload(args):
    cfg = dict(CONFIGS[args.config])
    if args.n:
        cfg["n"] = args.n
    return cfg


def config_json(cfg, world, extra=None):
    d = {"workload": f"{cfg['workload']} N={cfg['n']} ({args_config_name(cfg)})", "n": cfg["n"],
         "theta": cfg["theta"], "eps": cfg["eps"], "dt": cfg["dt"], "key_bits": cfg.get("key_bits", 16),
         "seed": cfg["seed"],
         "sort_every": cfg.get("sort_every", 1), "exchange": cfg.get("exchange", "none"),
         "balance": cfg.get("balance", "none"),
         "parallelism": "single" if world == 1 else f"hilbert-range x{world}",
         "l2": "inputs larger than L2 (bodies 320 MB + tree ~1 GB per step at N=1e7); no explicit flush"}
    if extra:
        d.update(extra)
    return d


def args_config_name(cfg):
    for k, v in CONFIGS.items():
        if v["workload"] == cfg["workload"] and v["seed"] == cfg["seed"]:
            return k
    return "custom"


# ------------------------------------------------------------- clocks ------
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.p = None
        self.lines = []

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                       "-lms", "50", "-i", str(self.idx)], stdout=subprocess.PIPE,
                                      stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.p = None

    def stop(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        rows = [[x.strip() for x in ln.split(",")] for ln in out.strip().splitlines() if ln.count(",") >= 8]
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        smax = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": reasons, "samples": len(rows),
                "power_w_max": max((float(r[3]) for r in rows if r[3].replace(".", "").isdigit()), default=None)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


def ncu_traffic(cfg, precision):
    """dram bytes per launch of the force kernel from a committed ncu --set
    full capture of THE SAME workload, N, theta and precision
    (profiles/*force_ncu*.json, newest first), else None."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "*force_ncu*.json")), reverse=True)
    for fn in files:
        try:
            with open(fn) as f:
                d = json.load(f)
        except (OSError, ValueError):
            continue
        c = d.get("config") or {}
        if (c.get("workload") == cfg["workload"] and c.get("n") == cfg["n"] and c.get("theta") == cfg["theta"]
                and c.get("precision", 32) == precision and c.get("multipole", 1) == 1
                and c.get("key_bits", 16) == cfg.get("key_bits", 16)):
            return {"bytes_per_launch": d.get("dram_bytes_per_launch"), "capture": os.path.basename(fn),
                    "captured_kernel_ms": float(d["metrics"]["gpu__time_duration.sum"])}
    return None


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                return ln.split(":", 1)[1].strip()
    except (OSError, subprocess.SubprocessError):
        pass
    return None


# ----------------------------------------------------------- CPU oracle ----
def cpu_oracle_sample(pos, vel, mass, cfg, target_seconds, seed=0):
    """The oracle as it stands on this host: full bbox/keys/stable-sort/
    permute/build on all N, forces for a bounded random sample of targets.
    Returns a dict: extrapolated full-step seconds, measured seconds of this
    sampled step, sample size, cores, interactions/s."""
    from oracle import oracle as O
    n = len(pos)
    rng = np.random.default_rng(seed)
    probe = np.sort(rng.choice(n, min(n, 500), replace=False))
    kb = cfg.get("key_bits", 16)
    t0 = time.perf_counter()
    prec = 64 if pos.dtype == np.float64 else 32
    r = O.step(pos, vel, mass, theta=cfg["theta"], eps=cfg["eps"], dt=cfg["dt"], key_bits=kb, integrate=False,
               targets=probe, precision=prec)
    t_all = time.perf_counter() - t0
    tf0 = time.perf_counter()
    r.tree.force(cfg["theta"], cfg["eps"], probe)
    t_probe = time.perf_counter() - tf0
    t_prep = max(0.0, t_all - t_probe)
    per_target = max(t_probe / len(probe), 1e-9)
    ns = int(min(n, max(len(probe), target_seconds / per_target)))
    targets = np.sort(rng.choice(n, ns, replace=False))
    tf0 = time.perf_counter()
    _, cnt = r.tree.force(cfg["theta"], cfg["eps"], targets)
    t_force = time.perf_counter() - tf0
    return {"t_full": t_prep + t_force * n / ns, "t_measured": t_all + t_probe + t_force, "t_prep": t_prep,
            "t_force": t_force, "ns": ns, "n": n, "cores": os.cpu_count(),
            "interactions_per_s": float(cnt.sum()) / t_force}


def cpu_desc(d):
    model = cpu_model()
    return (f"oracle (fp64 C++, g++ -O2, std::thread x {d['cores']}{', ' + model if model else ''}): full "
            f"bbox/keys/stable-sort/permute/build on N={d['n']} ({d['t_prep']:.1f} s) + forces for {d['ns']} random "
            f"targets ({d['t_force']:.1f} s); bodies/s = N / (prep + force time x N/{d['ns']})")


# ------------------------------------------------------------ reference ----
def run_reference(args, cfg, world, rank):
    """The reference arm of this tier: the oracle as it stands on the host
    cores.  Each step is a bounded sample of the workload (full preparation
    on all N, forces for a target sample); ms_per_step is the MEASURED wall
    time of such a sampled step, so ms_per_step x steps is this run's timed
    region; value (bodies/s) extrapolates each step's force time to all N
    targets (the rate of a full oracle step), stated in value_basis."""
    if rank != 0:
        return 0
    pos, vel, mass = generate(cfg["workload"], cfg["n"], cfg["seed"])
    meas, full, last = [], [], None
    per = min(args.cpu_seconds, 6.0)
    for i in range(args.warmup + args.steps):
        d = cpu_oracle_sample(pos, vel, mass, cfg, per, seed=i)
        if i >= args.warmup:
            meas.append(d["t_measured"])
            full.append(d["t_full"])
            last = d
    value = cfg["n"] / statistics.median(full)
    line = {"impl": "reference", "metric": metric_name(cfg), "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.mean(meas),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config_json(cfg, 1),
            "value_basis": "N / extrapolated full-step time (median over the timed sampled steps); ms_per_step is "
                           "the measured time of one sampled step",
            "extrapolated_ms_per_full_step": 1e3 * statistics.median(full),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": last["cores"], "kind": "oracle",
                             "sample": cpu_desc(last), "interactions_per_s": last["interactions_per_s"]},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ ours ----
def fp_peak(nsm, f64):
    peaks = measured_peaks()
    fmax = float(peaks.get("sm_max_mhz", 1965.0))
    lanes = 64 if f64 else 128  # FP64: 64 DFMA lanes/SM (measured 59/clk, scripts/micro/pipe_rates.cu)
    return 2 * lanes * nsm * fmax * 1e6 / 1e12, lanes, fmax


def force_timing(sim, reps):
    """K6's device time per launch, measured live with the library's CUDA
    events on the launching (context) stream, graphs off; plus the other
    stages' times of the same passes."""
    sim.set_option(5, 1)  # NBODY_OPT_TIMING
    sim.set_option(3, 0)  # NBODY_OPT_USE_GRAPH
    f_ms, f_int, stage = [], [], {}
    for _ in range(reps):
        sim.step(1)
        s2 = sim.stats()
        f_ms.append(s2["ms_force"])
        f_int.append(s2["interactions"])
        for k in ("ms_bbox_keys", "ms_sort", "ms_build", "ms_force", "ms_update"):
            stage.setdefault(k, []).append(s2[k])
    sim.set_option(3, 1)
    sim.set_option(5, 0)
    return statistics.median(f_ms), statistics.mean(f_int), {k: statistics.median(v) for k, v in stage.items()}


def timed_steps(sim, stream, steps, repeats, barrier):
    """Median over `repeats` of the device time of `steps` graph-replayed
    steps (CUDA events on the context stream)."""
    import torch
    out = []
    for _ in range(repeats):
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        sim.step(steps)
        e1.record(stream)
        barrier()
        out.append(e0.elapsed_time(e1))
    return out


def single_block(name, cfg, precision, steps, warmup, nsm):
    """An extra configuration timed inside the default run (one GPU): the
    same measurement as the headline, reported as a block of the line."""
    import torch
    from paper_conf_sc_casselldahg24_b200 import NBody
    f64 = precision == 64
    pos, vel, mass = generate(cfg["workload"], cfg["n"], cfg["seed"], np.float64 if f64 else np.float32)
    stream = torch.cuda.Stream()
    sim = NBody(cfg["n"], cfg["theta"], cfg["eps"], cfg["dt"], key_bits=cfg.get("key_bits", 16),
                stream=stream.cuda_stream, precision=precision)
    sim.set_bodies(pos, vel, mass)
    sim.step(warmup)

    def barrier():
        torch.cuda.synchronize()

    reps = timed_steps(sim, stream, steps, 3, barrier)
    ms = statistics.median(reps) / steps
    inter = int(sim.stats()["interactions"])
    force_ms, f_int, stage = force_timing(sim, 3)
    peak, lanes, fmax = fp_peak(nsm, f64)
    achieved = FLOPS_PER_INTERACTION * f_int / (force_ms / 1e3) / 1e12
    sim.close()
    return {"metric": metric_name(cfg), "config": config_json(dict(cfg, precision=precision), 1),
            "dtype": "f64" if f64 else "f32 (fp64 tree moments, key grid and opening test)",
            "ms_per_step": ms, "value": cfg["n"] / (ms / 1e3), "unit": UNIT, "steps": steps, "warmup": warmup,
            "repeats_ms": reps, "interactions_per_s": inter / (ms / 1e3), "interactions_per_body": inter / cfg["n"],
            "stage_ms": stage,
            "roofline": {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": ncu_traffic(cfg, precision), "kernel_ms": force_ms,
                         "kernel": "k_force (CALCULATEFORCE)",
                         "peak_basis": f"{'FP64' if f64 else 'FP32'} pipe 2 flop x {lanes} lanes x {nsm} SMs x "
                                       f"{fmax:.0f} MHz"}}


def calibration_block(sim, n, nsm, force_frac, nt=1 << 17):
    """NEXT-1 calibration: the fp32 all-pairs kernel (the same interaction
    arithmetic as K6, no traversal) on nt sampled targets against all n
    sources; its FP32-pipe fraction is the achievable ceiling K6 is compared
    with."""
    ids = np.sort(np.random.default_rng(11).choice(n, min(n, nt), replace=False))
    sim.allpairs_accel(ids[:4096], timed=True)  # warm-up
    ms = [sim.allpairs_accel(ids, timed=True)[1] for _ in range(2)]
    k_ms = min(ms)
    peak, lanes, fmax = fp_peak(nsm, False)
    inter = float(len(ids)) * n
    achieved = FLOPS_PER_INTERACTION * inter / (k_ms / 1e3) / 1e12
    frac = achieved / peak
    return {"kernel": "k_allpairs32 (NEXT-1 All-Pairs, fp32, Nyland-tiled)", "targets": len(ids), "sources": n,
            "kernel_ms": k_ms, "interactions_per_s": inter / (k_ms / 1e3), "achieved": achieved, "peak": peak,
            "unit": "TFLOP/s", "frac": frac, "k6_frac_over_allpairs_frac": force_frac / frac}


def run_ours(args, cfg, world, rank, local):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_casselldahg24_b200 import NBody

    # NBODY_BENCH_ONE_DEVICE=1 (validation of the N > 1 path on a one-GPU
    # box only, never a reported number): every rank on GPU 0, gloo for the
    # host-side plumbing; the exchange itself still runs over CUDA IPC.
    one_device = world > 1 and os.environ.get("NBODY_BENCH_ONE_DEVICE") == "1"
    if one_device:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if one_device:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    n = cfg["n"]
    cfg["key_bits"] = args.key_bits
    f64 = args.precision == 64
    pos, vel, mass = generate(cfg["workload"], n, cfg["seed"], np.float64 if f64 else np.float32)
    stream = torch.cuda.Stream()
    sim = NBody(n, cfg["theta"], cfg["eps"], cfg["dt"], key_bits=args.key_bits, stream=stream.cuda_stream,
                precision=args.precision)
    cfg["precision"] = args.precision
    if args.sort_every != 1:
        sim.set_option(7, args.sort_every)  # NBODY_OPT_SORT_EVERY
        cfg["sort_every"] = args.sort_every
    use_peer = world > 1 and args.exchange == "peer" and world <= 8
    if use_peer and not one_device:
        # every rank must reach every other rank's GPU by loads/stores (NVLink /
        # NVSwitch P2P); decided collectively so that all ranks pick the same
        # exchange, else the NCCL all-gather on torch's communicator
        devs = [None] * world
        dist.all_gather_object(devs, local)
        ok = all(d == local or torch.cuda.can_device_access_peer(local, d) for d in devs)
        flag = torch.tensor([1 if ok else 0], device="cuda")
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if not int(flag.item()):
            use_peer = False
            cfg["exchange_note"] = "no peer access between the ranks' GPUs: NCCL all-gather instead"
    if world > 1:
        if use_peer:
            sim.attach_peers_group(rank, world)
            if args.balance == "cost":
                sim.set_option(9, 1)  # NBODY_OPT_BALANCE
            cfg["balance"] = args.balance
        elif one_device:
            sim.attach_process_group(rank, world)
        else:  # NCCL all-gather on torch.distributed's own communicator
            sim.attach_torch_comm()
        cfg["exchange"] = sim.exchange_mode()
    sim.set_bodies(pos, vel, mass)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    sim.step(args.warmup)
    reps = timed_steps(sim, stream, args.steps, max(1, args.repeats), barrier)
    clk = clocks.stop()
    if world > 1:  # max over ranks, per repeat
        t = torch.tensor(reps, device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        reps = [float(x) for x in t.tolist()]
    ms = statistics.median(reps) / args.steps
    st = sim.stats()
    inter = int(st["interactions"])  # last step, owned targets of this rank
    if world > 1:
        t = torch.tensor([inter], device="cuda", dtype=torch.float64)
        dist.all_reduce(t)
        inter = int(t.item())
    launches = int(st["kernels_per_step"]) * args.steps

    # Dominant kernel (K6 force): its device time per launch, measured live
    # with CUDA events on the launching stream, graphs off.
    force_ms, f_int, stage = force_timing(sim, max(3, min(args.steps, 5)))
    nsm = torch.cuda.get_device_properties(local).multi_processor_count
    peak_tflops, lanes, fmax = fp_peak(nsm, f64)
    achieved = FLOPS_PER_INTERACTION * f_int / (force_ms / 1e3) / 1e12
    roofline = {"bound": "alu", "achieved": achieved, "peak": peak_tflops, "unit": "TFLOP/s",
                "frac": achieved / peak_tflops, "traffic": ncu_traffic(cfg, args.precision),
                "kernel": "k_force (CALCULATEFORCE)", "flops_per_interaction": FLOPS_PER_INTERACTION,
                "kernel_ms": force_ms,
                "peak_basis": f"{'FP64' if f64 else 'FP32'} pipe 2 flop x {lanes} lanes x {nsm} SMs x {fmax:.0f} MHz "
                              "(sm_max, MEASURED_PEAKS.json; guide unit counts, no FP32 figure is measured there)",
                "share_of_step": force_ms / ms}

    # End to end through the public API: pinned host inputs -> step -> host result.
    e2e = None
    if not args.no_e2e:
        hp = torch.from_numpy(pos).pin_memory()
        hv = torch.from_numpy(vel).pin_memory()
        hm = torch.from_numpy(mass).pin_memory()
        outs = [torch.empty((n, 3), dtype=torch.float64 if f64 else torch.float32).pin_memory() for _ in range(2)]
        # every rank loads the full input and reads the full result (the state
        # is replicated after each step's exchange).  fp32: the pipelined
        # calls, so step k's copies overlap the neighbouring steps' kernels
        # (copy stream, double-buffered staging); FP64 mode: synchronous calls.
        if f64:
            def e2e_step(k):
                sim.set_bodies(hp, hv, hm)
                sim.step(1)
                sim.get_positions64(outs[k & 1])
        else:
            def e2e_step(k):
                sim.set_bodies_async(hp, hv, hm)
                sim.step(1)
                sim.get_positions_async(outs[k & 1])
        for k in range(2):
            e2e_step(k)
        sim.sync()
        barrier()
        t0 = time.perf_counter()
        for k in range(args.steps):
            e2e_step(k)
        sim.sync()
        barrier()
        e2e_ms = 1e3 * (time.perf_counter() - t0) / args.steps
        if world > 1:
            from paper_conf_sc_casselldahg24_b200.dist import max_over_ranks
            e2e_ms = max_over_ranks(e2e_ms, device="cuda")
        w = 2 if f64 else 1
        e2e = {"value": n / (e2e_ms / 1e3), "unit": UNIT, "h2d_bytes_per_step": 28 * w * n * world,
               "d2h_bytes_per_step": 12 * w * n * world, "ms_per_step": e2e_ms,
               "path": ("nbody_set_bodies64 + nbody_step(1) + nbody_get_positions64 (pinned host), per rank" if f64
                        else "nbody_set_bodies_async(pinned host) + nbody_step(1) + nbody_get_positions_async(pinned "
                             "host) per step, copies on the copy stream overlapping the neighbouring steps, "
                             "nbody_sync at the end; per rank")}

    extras = {}
    if world == 1 and not args.no_extras and not f64 and args.config == "cfg3" and not args.n:
        try:
            extras["calibration"] = calibration_block(sim, n, nsm, roofline["frac"])
        except Exception as ex:  # noqa: BLE001 -- an extra block never sinks the headline
            extras["calibration"] = {"error": repr(ex)}
    sim.close()
    if world == 1 and not args.no_extras and not f64 and args.config == "cfg3" and not args.n:
        for key, c, prec in (("fp64", dict(cfg), 64), ("cfg2", dict(CONFIGS["cfg2"], key_bits=16), 32)):
            try:
                extras[key] = single_block(key, c, prec, args.steps, args.warmup, nsm)
            except Exception as ex:  # noqa: BLE001
                extras[key] = {"error": repr(ex)}
        extras["fp64"]["note"] = ("the paper's own precision (FP64 throughout, P:272, P:282) on the headline "
                                  "workload; roofline against the FP64 pipe") if "error" not in extras["fp64"] else None

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        d = cpu_oracle_sample(pos, vel, mass, cfg, args.cpu_seconds)
        cpu = {"value": n / d["t_full"], "unit": UNIT, "cores": d["cores"], "kind": "oracle", "sample": cpu_desc(d),
               "interactions_per_s": d["interactions_per_s"], "cpu_model": cpu_model()}

    if rank == 0:
        line = {"metric": metric_name(cfg), "value": n / (ms / 1e3), "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None,
                "dtype": "f64" if f64 else "f32 (fp64 tree moments, key grid and opening test)",
                "data": "synthetic", "impl": "ours",
                "config": config_json(cfg, world, {"repeats": len(reps)}),
                "repeats_ms": reps,
                "interactions_per_s": inter / (ms / 1e3), "interactions_per_body": inter / n,
                "stage_ms": stage,
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
                "clocks": clk, **extras}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    world, rank, local = dist_env()
    cfg = workload(args)
    if args.impl == "reference":
        return run_reference(args, cfg, world, rank)
    return run_ours(args, cfg, world, rank, local)


if __name__ == "__main__":
    sys.exit(main())
