#!/usr/bin/env python
"""MemXCT hot-path benchmark (BASELINE.json metric: CG iter/s and SpMV GFLOP/s + HBM GB/s).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--iters 30]
    python bench.py --impl reference ...        # the fp64 CPU oracle, timed on host cores

One STEP = one CGLS reconstruction (`--iters` iterations, default 30 = the paper's count,
P:957) of one synthetic slice: the whole hot path of SURVEY 8(a) a7-a10 (forward SpMV + back
SpMV + fused vector steps per iteration, plus the setup backprojection), launched as one CUDA
graph through the C ABI (memxct_cg).  The matrices are built once (memxct_build, preprocessing
a1-a6) before timing, as in the paper.

value = CG iterations per second over the whole job; inputs resident in HBM.  The 11.8 GB
matrix stream per SpMV (cfg 3) is ~90x the L2, so no flush is needed between steps.
e2e = the same metric through memxct_cg_host (pinned host sinogram in, host tomogram out).
roofline = the SpMV kernel (both directions), algorithmic bytes per launch
over its CUDA-event duration, against MEASURED_PEAKS.json's HBM copy bandwidth.

N > 1 (torchrun): the slice is domain-decomposed over the ranks (A = R C A_p): each
GPU owns Hilbert tile ranges of the tomogram and sinogram, partial sinograms move by NCCL grouped
send/recv, CG dots by allreduce (strong scaling); the max over ranks of the device time is taken.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only if MEASURED_PEAKS.json is absent


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--iters", type=int, default=30)
    ap.add_argument("--part-rows", type=int, default=None)
    ap.add_argument("--buffer", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true",
                    help="skip the MIXED+CANONICAL, preprocessing and multi-slice side measurements")
    ap.add_argument("--cpu-sample", type=float, default=0.05,
                    help="fraction of the config's rays the oracle baseline traces and times")
    ap.add_argument("--cpu-full", action="store_true",
                    help="oracle baseline on the WHOLE config (cfg3: ~30 GB host RAM, minutes)")
    ap.add_argument("--spmv-reps", type=int, default=20)
    ap.add_argument("--slices", type=int, default=8, help="multi-slice batch measured beside the headline (1 = off)")
    ap.add_argument("--variant", default=None, choices=["peer", "dense"], help=argparse.SUPPRESS)
    ap.add_argument("--distributed", action="store_true",
                    help="run the decomposed path (NCCL communicator, exchange, allreduce) even at N = 1")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "host"],
                    help="N > 1 transport: nccl (one GPU per rank) or host (memxct_plan_set_comm_host: "
                         "processes may share a GPU -- exercises the multi-rank bench on one GPU; "
                         "its times are not multi-GPU numbers)")
    return ap.parse_args()


def _dist_allreduce_max(t):
    """MAX over ranks of a CUDA tensor (through the CPU on gloo)."""
    import torch.distributed as dist
    if dist.get_backend() == "gloo":
        c = t.cpu()
        dist.all_reduce(c, op=dist.ReduceOp.MAX)
        t.copy_(c)
    else:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t


def _dist_allgather(t):
    import torch
    import torch.distributed as dist
    src = t.cpu() if dist.get_backend() == "gloo" else t
    out = [torch.empty_like(src) for _ in range(dist.get_world_size())]
    dist.all_gather(out, src)
    return torch.stack(out).cpu()


def _device_index(args):
    import torch
    local = int(os.environ.get("LOCAL_RANK", 0))
    return local % max(1, torch.cuda.device_count()) if args.transport == "host" else local


def workload_name(cfg, iters):
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    n, m, c = inputs.CONFIGS[cfg]
    return (f"cfg{cfg}: {n}x{n} tomogram, {m} projections x {c} channels, modified Shepp-Logan "
            f"sinogram, {iters}-iteration CGLS per step")


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


# ------------------------------------------------------------------------------------------
# clocks sampler (B200_PROFILING.md "clocks line")
# ------------------------------------------------------------------------------------------
class Clocks:
    FIELDS = ["clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": float(max(mx)) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------------
# the oracle (CPU baseline / reference arm): bounded sample of the same workload
# ------------------------------------------------------------------------------------------
def host_info():
    """Host cores and CPU model (nproc / lscpu) of the box the oracle runs on."""
    model = ""
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.lower().startswith("model name"):
                model = ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def oracle_sample(cfg, frac, seed=0):
    """Trace a random `frac` of the config's rays with the oracle (orc_sample_rows, untimed) and
    build the CSR of those rows of A and of their transpose (rows = pixels); returns a dict."""
    import oracle
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    n, m, c = inputs.CONFIGS[cfg]
    rng = np.random.default_rng(seed)
    if frac >= 1.0:
        rays = np.arange(m * c, dtype=np.int64)
    else:
        rays = np.sort(rng.choice(m * c, max(1, int(frac * m * c)), replace=False)).astype(np.int64)
    t0 = time.perf_counter()
    ptr, pix, ln = oracle.sample_rows(n, m, c, rays)
    t_trace = time.perf_counter() - t0
    tp, tc, tv = oracle.csr_transpose(ptr, pix, ln, n * n)    # A^T restricted to the sampled rays
    return {"ptr": ptr, "cols": pix, "vals": ln, "tptr": tp, "tcols": tc, "tvals": tv,
            "nrays": len(rays), "npix": n * n, "nnz": len(pix), "trace_s": t_trace, "frac": frac}


def oracle_step(sample, threads):
    """One oracle step on the sample: forward + back threaded CSR SpMV (orc_spmv_csr_threaded,
    rows split over `threads` host threads; 1 = the plain single-thread product).  Returns
    (seconds, threads used)."""
    import oracle
    x = np.ones(sample["npix"])
    y = np.ones(sample["nrays"])
    t0 = time.perf_counter()
    _, nt = oracle.spmv_csr_threaded(sample["ptr"], sample["cols"], sample["vals"], x, threads)
    oracle.spmv_csr_threaded(sample["tptr"], sample["tcols"], sample["tvals"], y, threads)
    return time.perf_counter() - t0, nt


def nnz_model(cfg):
    from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
    n, m, c = inputs.CONFIGS[cfg]
    return int(round(1.1953 * m * n * n))


def cpu_baseline(cfg, nnz_full, frac=0.05, reps=3):
    """the oracle on the box's host cores -- a threaded CSR SpMV over all cores and
    the single-thread product -- on a bounded random ray sample of the workload, forward + back
    per CG iteration, extrapolated by nnz (the work is proportional to nnz)."""
    sample = oracle_sample(cfg, frac)
    scale = nnz_full / max(1, sample["nnz"])
    res = {}
    for threads in (0, 1):
        best, nt = None, 1
        for _ in range(reps):
            dt, nt = oracle_step(sample, threads)
            best = dt if best is None else min(best, dt)
        res[threads] = (1.0 / (best * scale), nt, best)
    hi = host_info()
    full = sample["frac"] >= 1.0
    return {"value": res[0][0], "unit": "CG iter/s", "cores": res[0][1], "kind": "oracle",
            "single_thread": {"value": res[1][0], "unit": "CG iter/s", "cores": 1,
                              "fwd_back_s_sample": res[1][2]},
            "threaded_fwd_back_s_sample": res[0][2],
            "host": hi,
            "sample": (f"{'all' if full else 'a random %.0f%% of the' % (100 * sample['frac'])} rays of cfg{cfg} "
                       f"({sample['nrays']} rays, {sample['nnz']} nonzeros) traced by orc_sample_rows "
                       f"({sample['trace_s']:.1f} s, untimed); timed: forward + back orc_spmv_csr_threaded "
                       f"on them, best of {reps}, all {res[0][1]} host threads (value) and 1 thread "
                       f"(single_thread); CG iter/s = 1 / (t x nnz_full / nnz_sample)"
                       + ("" if full else f", x{scale:.1f}"))}


def run_reference(args, rank, world):
    """The reference arm: the oracle as it stands (threaded CSR SpMV on all host cores) on a
    bounded sample of the workload; rank 0 only."""
    if rank != 0:
        return
    cfg = args.config
    nnz_full = nnz_model(cfg)
    sample = oracle_sample(cfg, args.cpu_sample)
    nt = 1
    for _ in range(args.warmup):
        oracle_step(sample, 0)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        _, nt = oracle_step(sample, 0)
    dt = time.perf_counter() - t0
    # each step does forward + back over nnz_sample of the nnz_full of one CG iteration
    value = args.steps * sample["nnz"] / nnz_full / dt
    hi = host_info()
    desc = (f"{sample['nrays']} random rays ({100 * sample['frac']:.0f}%) of cfg{cfg}, {sample['nnz']} "
            f"nonzeros; forward + back orc_spmv_csr_threaded per step on {nt} host threads "
            f"({hi['cpu_model']}), extrapolated to full nnz")
    line = {
        "impl": "reference", "metric": "CG iter/s", "value": value, "unit": "CG iter/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(cfg, args.iters) + " (oracle: ray sample, "
                   "forward + back SpMV per step, extrapolated to full nnz)"},
        "cpu_baseline": {"value": value, "unit": "CG iter/s", "cores": nt, "kind": "oracle",
                         "sample": desc, "host": hi},
        "e2e": {"value": value, "unit": "CG iter/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------
def spmv_bytes(info):
    """Algorithmic bytes of one SpMV: 6 B per nonzero (uint16
    local index + fp32 value), 8 B per stage-map entry (int32 map + fp32 gather),
    4 B per output row written.  Padding slots are not counted."""
    return 6 * info["nnz"] + 8 * info["map_entries"] + 4 * info["rows"]


def bench_multislice(args, plan1, y1, n, m, c, stream):
    """K slices of the same geometry share one matrix stream (SpMM).  A
    separate plan tuned for K slices (MEMXCT_OPT_SLICES) runs K independent 30-iteration CGLS
    solves per step; reported as slice-iterations per second next to the single-slice value."""
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    K = args.slices
    del plan1
    plan = MemXCT(n, m, c, slices=K).build()
    Y = y1.unsqueeze(0).repeat(K, 1).contiguous()
    Y *= torch.linspace(0.5, 1.5, K, device=Y.device).unsqueeze(1)  # K different slices
    X = torch.empty(K, n * n, dtype=torch.float32, device=Y.device)
    for _ in range(max(1, args.warmup)):
        plan.cg_batch(Y, args.iters, x=X, stream=stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    steps = max(1, args.steps // 2)
    e0.record(stream)
    for _ in range(steps):
        plan.cg_batch(Y, args.iters, x=X, stream=stream)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    # SpMM alone (both directions), per launch
    XB = torch.empty_like(X)
    YB = torch.empty_like(Y)
    reps = 10
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 * reps + 1)]
    ev[0].record(stream)
    for i in range(reps):
        plan.forward_batch(X, YB, stream=stream)
        ev[2 * i + 1].record(stream)
        plan.back_batch(Y, XB, stream=stream)
        ev[2 * i + 2].record(stream)
    torch.cuda.synchronize()
    tf = float(np.median([ev[2 * i].elapsed_time(ev[2 * i + 1]) for i in range(reps)]))
    tb = float(np.median([ev[2 * i + 1].elapsed_time(ev[2 * i + 2]) for i in range(reps)]))
    fi = plan.layout_info(0)
    out = {"slices": K, "value": K * args.iters * steps / (ms * 1e-3), "unit": "slice CG iter/s",
           "ms_per_step": ms / steps, "spmm_fwd_ms": tf, "spmm_back_ms": tb,
           "fwd_gflops": 2 * K * fi["nnz"] / (tf * 1e-3) / 1e9,
           "buffer_entries": plan.get_option("buffer_entries"),
           "note": "K independent 30-iteration CGLS solves per step sharing one matrix stream per "
                   "SpMM; each slice bit-identical to its single-slice solve (tests)"}
    plan.close()
    return out


def bench_mixed_canonical(args, n, m, c, ph, stream):
    """The parity-gated mode (reading R16: PRECISION = MIXED, CANONICAL = 1 -- fp64 vectors and
    one fp64 fma chain per row in Hilbert order, dots as fixed chains; its 30-iteration image is
    bit-identical to the canonical oracle's), timed like the headline: `steps` CGLS solves of the
    same slice.  The matrix stream is the same 6 B per nonzero as FP32."""
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    plan = MemXCT(n, m, c, precision="mixed", canonical=True).build()
    y = plan.forward(torch.from_numpy(ph.astype(np.float64)).cuda())
    x = torch.empty(plan.local_size(0), dtype=torch.float64, device=y.device)
    for _ in range(max(1, args.warmup)):
        plan.cg(y, args.iters, x=x, stream=stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        plan.cg(y, args.iters, x=x, stream=stream)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    sp = plan.spmv_time(10, stream=stream)
    fi, bi = plan.layout_info(0), plan.layout_info(1)
    out = {"value": args.iters * args.steps / (ms * 1e-3), "unit": "CG iter/s", "ms_per_step": ms / args.steps,
           "spmv_fwd_ms": sp["fwd_us"] * 1e-3, "spmv_back_ms": sp["back_us"] * 1e-3,
           "spmv_gbs": (spmv_bytes(fi) + spmv_bytes(bi)) / ((sp["fwd_us"] + sp["back_us"]) * 1e-6) / 1e9,
           "buffer_entries_fp64": [fi["buffer_entries"], bi["buffer_entries"]],
           "note": "PRECISION=MIXED, CANONICAL=1: the mode the 1e-3 x_30 gate binds (bit-identical to "
                   "the canonical oracle in tests); same matrix bytes as FP32"}
    plan.close()
    return out


PAPER_PREPROC = {  # per node, the paper's Tables 4-5: context, other hardware
    "ADS2": {"shape": (512, 750, 512), "paper_s": 4.00, "paper_hw": "1 KNL (Theta), Table 4"},
    "RDS1": {"shape": (2048, 1501, 2048), "paper_s": 139.0, "paper_hw": "1 KNL (Theta), Table 5 (146.3 s in Table 4)"},
}


def bench_preprocessing(args, plan, build_s):
    """preprocessing throughput (memxct_build: Hilbert ordering, Siddon
    tracing, transposition, buffered layouts) per phase -- the bench config's build, and fresh
    builds at the paper's ADS2 (750 x 512) and RDS1 (1501 x 2048) shapes, whose single-node
    preprocessing the paper times at 4.00 s and 139 s on one KNL."""
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT
    out = {f"cfg{args.config}": {"build_s": build_s, "phases_s": plan.build_phases(),
                                 "nnz": plan.stats()["nnz"]}}
    for name, d in PAPER_PREPROC.items():
        n, m, c = d["shape"]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        p = MemXCT(n, m, c).build()
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        out[name] = {"shape": {"n": n, "projections": m, "channels": c}, "build_s": wall,
                     "phases_s": p.build_phases(), "nnz": p.stats()["nnz"],
                     "nnz_per_s": p.stats()["nnz"] / wall,
                     "paper_s": d["paper_s"], "paper_hw": d["paper_hw"]}
        p.close()
        del p
    return out


def variant_child(args):
    """Child process of bench_exchange_variant: one rank of the same job on its own NCCL
    communicator (a fresh rendezvous), the CG with exchange `args.variant`; rank 0 prints one
    JSON line."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, bootstrap_host_comm_name, bootstrap_unique_id, inputs
    local = _device_index(args)
    torch.cuda.set_device(local)
    dist.init_process_group("gloo" if args.transport == "host" else "nccl")
    rank, world = dist.get_rank(), dist.get_world_size()
    n, m, c = inputs.CONFIGS[args.config]
    if args.transport == "host":
        comm = {"host_comm": bootstrap_host_comm_name(rank)}
    else:
        comm = {"unique_id": bootstrap_unique_id(rank)}
    plan = MemXCT(n, m, c, rank=rank, nranks=world, device=local, vector_order="plan", exchange=args.variant,
                  **comm).build()
    ph = np.ascontiguousarray(inputs.shepp_logan(n).astype(np.float32)[plan.local_indices(0)])
    stream = torch.cuda.current_stream()
    y = plan.forward(torch.from_numpy(ph).cuda())
    x = torch.empty(plan.local_size(0), dtype=torch.float32, device=y.device)
    for _ in range(max(1, args.warmup)):
        plan.cg(y, args.iters, x=x, stream=stream)
    dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        plan.cg(y, args.iters, x=x, stream=stream)
    e1.record(stream)
    torch.cuda.synchronize()
    ex = plan.exchange_time(20, stream=stream) if args.variant == "dense" else {"fwd_us": 0.0, "back_us": 0.0}
    t = torch.tensor([e0.elapsed_time(e1), ex["fwd_us"], ex["back_us"]], dtype=torch.float64, device=y.device)
    _dist_allreduce_max(t)
    out = {"value": args.iters * args.steps / (float(t[0]) * 1e-3), "unit": "CG iter/s",
           "ms_per_step": float(t[0]) / args.steps}
    if args.variant == "dense":
        out["exchange_us_per_cg_iter"] = float(t[1] + t[2])
    plan.close()
    dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(out), flush=True)


def bench_exchange_variant(args, rank, world, kind):
    """N > 1: the same CG with another exchange, reported beside the NCCL all-to-allv headline:
    "peer" = EXCHANGE 1 (SpMV epilogue / pack kernel store straight into the peers' buffers over
    NVLink, CG dots over peer memory, NEXT-2); "dense" = EXCHANGE 2 (reduce-scatter / allgather of
    the whole partial sinogram, SURVEY 8(e)'s comparison).  Every rank runs it in a child process
    with its own rendezvous, so a failure there (a peer-flag wait traps after ~20 s instead of
    hanging) is reported without taking down the headline's process."""
    env = dict(os.environ)
    env["MASTER_PORT"] = str(int(os.environ.get("MASTER_PORT", "29500")) + (17 if kind == "peer" else 23))
    # under torchrun the ranks' env:// rendezvous is a client of the agent's store; the children's
    # fresh rendezvous needs its own store, hosted by child rank 0 (else every child waits for a
    # server that never starts -- the r02l host-transport run timed out exactly so)
    env.pop("TORCHELASTIC_USE_AGENT_STORE", None)
    cmd = [sys.executable, os.path.abspath(__file__), "--variant", kind, "--config", str(args.config),
           "--iters", str(args.iters), "--steps", str(args.steps), "--warmup", str(args.warmup),
           "--transport", args.transport]
    try:
        r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=300)
    except subprocess.TimeoutExpired:
        return {"error": "timed out after 300 s"}
    if rank != 0:
        return None
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    if r.returncode != 0 or not lines:
        return {"error": f"exit {r.returncode}: " + (r.stderr.strip().splitlines() or [""])[-1][:300]}
    return json.loads(lines[-1])


def run_ours(args, rank, world):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs, kernel_launch_count

    local = _device_index(args)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = args.config
    n, m, c = inputs.CONFIGS[cfg]
    kw = {}
    if args.part_rows:
        kw["part_rows"] = args.part_rows
    if args.buffer:
        kw["buffer_entries"] = args.buffer
    dist_mode = world > 1 or args.distributed
    t0 = time.perf_counter()
    if dist_mode:
        # domain decomposition over the ranks (A = R C A_p), NCCL exchange
        from paper_conf_sc_hidayetoglubgrg19_b200 import bootstrap_host_comm_name, bootstrap_unique_id
        if args.transport == "host":
            kw["host_comm"] = bootstrap_host_comm_name(rank)
        else:
            kw["unique_id"] = bootstrap_unique_id(rank)
        plan = MemXCT(n, m, c, rank=rank, nranks=world, device=local, vector_order="plan", **kw).build()
    else:
        plan = MemXCT(n, m, c, **kw).build()
    torch.cuda.synchronize()
    build_s = time.perf_counter() - t0
    st = plan.stats()
    fi, bi = plan.layout_info(0), plan.layout_info(1)

    # synthetic slice: phantom sinogram from our own forward projection (values do not change
    # the access pattern; the parity tests pin the values against the oracle)
    ph = inputs.shepp_logan(n).astype(np.float32)
    if dist_mode:
        ph = np.ascontiguousarray(ph[plan.local_indices(0)])
    x_ph = torch.from_numpy(ph).to(dev)
    y = plan.forward(x_ph)
    x = torch.empty(plan.local_size(0), dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()

    for _ in range(args.warmup):
        plan.cg(y, args.iters, x=x, stream=stream)
    torch.cuda.synchronize()

    clocks = Clocks(local)
    clocks.start()
    time.sleep(0.3)
    if dist_mode:
        dist.barrier()
    torch.cuda.synchronize()
    k0 = kernel_launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        plan.cg(y, args.iters, x=x, stream=stream)
    ev1.record(stream)
    torch.cuda.synchronize()
    launches = kernel_launch_count() - k0
    ms = ev0.elapsed_time(ev1)

    # SpMV kernels alone, each launch bracketed by events on the launching stream.  N > 1: the
    # rank's A_p / A_p^T kernels without the exchange (memxct_spmv_time, CUDA events on this
    # stream), so the roofline is the kernel's; the exchange is timed separately below.
    fwd_ms, back_ms = [], []
    if dist_mode:
        sp_t = plan.spmv_time(args.spmv_reps, stream=stream)
        fwd_ms, back_ms = [sp_t["fwd_us"] * 1e-3], [sp_t["back_us"] * 1e-3]
    else:
        yb = torch.empty_like(y)
        xb = torch.empty_like(x)
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(2 * args.spmv_reps + 1)]
        evs[0].record(stream)
        for i in range(args.spmv_reps):
            plan.forward(x, yb, stream=stream)
            evs[2 * i + 1].record(stream)
            plan.back(y, xb, stream=stream)
            evs[2 * i + 2].record(stream)
        torch.cuda.synchronize()
        for i in range(args.spmv_reps):
            fwd_ms.append(evs[2 * i].elapsed_time(evs[2 * i + 1]))
            back_ms.append(evs[2 * i + 1].elapsed_time(evs[2 * i + 2]))
    clk = clocks.stop()
    # per-rank kernel times and algorithmic bytes (one row per rank at N > 1)
    per_rank = torch.tensor([float(np.median(fwd_ms)), float(np.median(back_ms)),
                             spmv_bytes(fi), spmv_bytes(bi), fi["nnz"], bi["nnz"]],
                            dtype=torch.float64, device=dev)
    if dist_mode:
        per_rank_all = _dist_allgather(per_rank).numpy()
    else:
        per_rank_all = per_rank.cpu().numpy()[None, :]

    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if dist_mode:
        _dist_allreduce_max(t)
    ms_max = float(t.item())

    # e2e through the C ABI with host buffers (pinned sinogram in, tomogram out)
    y_host = torch.empty(plan.local_size(1), dtype=torch.float32, pin_memory=True)
    y_host.copy_(y.cpu())
    x_host = torch.empty(plan.local_size(0), dtype=torch.float32, pin_memory=True)
    plan.cg_host_ptr(y_host.data_ptr(), x_host.data_ptr(), args.iters, stream=stream)  # warm
    if dist_mode:
        dist.barrier()
    te0 = time.perf_counter()
    for _ in range(args.steps):
        plan.cg_host_ptr(y_host.data_ptr(), x_host.data_ptr(), args.iters, stream=stream)
    te = time.perf_counter() - te0
    te_t = torch.tensor([te], dtype=torch.float64, device=dev)
    if dist_mode:
        _dist_allreduce_max(te_t)
    te = float(te_t.item())

    exch_t = None
    if dist_mode:
        exch_t = plan.exchange_time(20, stream=stream)
        et = torch.tensor([exch_t["fwd_us"], exch_t["back_us"]], dtype=torch.float64, device=dev)
        _dist_allreduce_max(et)
        exch_t = {"fwd_us": float(et[0]), "back_us": float(et[1]),
                  "per_cg_iter_us": float(et[0] + et[1]),
                  "local_spmv_fwd_us": float(per_rank_all[:, 0].max() * 1e3),
                  "local_spmv_back_us": float(per_rank_all[:, 1].max() * 1e3),
                  "how": "max over ranks, CUDA events, 20 reps (memxct_exchange_time: C + R forward, "
                         "R^T + C^T back, no SpMV); local_spmv = A_p / A_p^T kernels alone"}

    peer = dense = None
    if dist_mode:
        dist.barrier()
        peer = bench_exchange_variant(args, rank, world, "peer")
        dense = bench_exchange_variant(args, rank, world, "dense")
        dist.barrier()

    multislice = mixed = prep = None
    if not dist_mode and not args.no_extras:
        prep = bench_preprocessing(args, plan, build_s)
        mixed = bench_mixed_canonical(args, n, m, c, ph, stream)
        if args.slices > 1:
            multislice = bench_multislice(args, plan, y, n, m, c, stream)

    if rank != 0:
        return
    from paper_conf_sc_hidayetoglubgrg19_b200.memxct import read_ceiling
    read_gbs = read_ceiling(8_000_000_000, 20, stream=stream)  # live, same GPU, after the timed region
    hbm_peak, peak_src = peaks()
    # dominant kernel = the SpMV pair of the slowest rank (the one every CG iteration waits for)
    slow = int(np.argmax(per_rank_all[:, 0] + per_rank_all[:, 1]))
    tf, tb = per_rank_all[slow, 0] * 1e-3, per_rank_all[slow, 1] * 1e-3
    fb, bb = per_rank_all[slow, 2], per_rank_all[slow, 3]
    fnnz, bnnz = per_rank_all[slow, 4], per_rank_all[slow, 5]
    achieved = (fb + bb) / (tf + tb) / 1e9
    traffic = None
    prof = os.path.join(ROOT, "profiles", f"ncu_spmv_cfg{cfg}.json")
    if os.path.exists(prof):
        with open(prof) as f:
            traffic = json.load(f).get("traffic_bytes_per_launch")
    iters_total = args.iters * args.steps  # one slice, decomposed over all ranks
    value = iters_total / (ms_max * 1e-3)
    line = {
        "metric": "CG iter/s", "value": value, "unit": "CG iter/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": workload_name(cfg, args.iters),
                   "l2": "no flush: the matrix stream per SpMV (%.1f GB) exceeds the 126 MB L2" %
                         (6 * st["stored_slots"] / 2 / 1e9),
                   "part_rows": plan.get_option("part_rows"),
                   "buffer_entries": plan.get_option("buffer_entries"),
                   "parallelism": ((f"domain decomposition over {world} GPUs (A = R C A_p, NCCL all-to-allv)"
                                    if args.transport == "nccl" else
                                    f"domain decomposition over {world} processes sharing "
                                    f"{torch.cuda.device_count()} GPU(s) (host transport; NOT a multi-GPU timing)")
                                   if dist_mode else "single GPU")},
        "spmv": {"fwd_ms": tf * 1e3, "back_ms": tb * 1e3,
                 "fwd_gflops": 2 * fnnz / tf / 1e9, "back_gflops": 2 * bnnz / tb / 1e9,
                 "rank": slow,
                 "how": ("slowest rank's A_p / A_p^T kernels alone (memxct_spmv_time), exchange excluded"
                         if dist_mode else "forward / back SpMV launches, CUDA events, median"),
                 "fwd_gbs": fb / tf / 1e9, "back_gbs": bb / tb / 1e9,
                 "nnz": st["nnz"], "stored_slots_per_dir": [fi["slots"], bi["slots"]],
                 "padding": [fi["slots"] / fi["nnz"] - 1, bi["slots"] / bi["nnz"] - 1],
                 "map_entries": [fi["map_entries"], bi["map_entries"]],
                 "stored_bytes_per_dir": [6 * fi["slots"] + 4 * fi["map_entries"],
                                          6 * bi["slots"] + 4 * bi["map_entries"]]},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                     "frac": achieved / hbm_peak, "traffic": traffic, "peak_source": peak_src,
                     "kernel": "spmv_f32_kernel (forward A + back A^T, per launch)" +
                               (f"; rank {slow}'s A_p + A_p^T, the slowest of {world}" if dist_mode else ""),
                     "algorithmic_bytes_per_launch": [fb, bb],
                     "read_ceiling": {"gbs": read_gbs, "frac": achieved / read_gbs,
                                      "how": "memxct_read_ceiling: 8 GB read-only stream with the SpMV's "
                                             "16 B ld.global.nc evict-first load, grid-stride over all SMs, "
                                             "best of 3 launch shapes (the peak above is a read+write copy)"}},
        "clocks": clk,
        "e2e": {"value": iters_total / te, "unit": "CG iter/s",
                "h2d_bytes_per_step": 4 * plan.local_size(1), "d2h_bytes_per_step": 4 * plan.local_size(0)},
        "gpu_launches": launches,
        "build_s": build_s,
        "device_bytes": st["device_bytes"],
    }
    if dist_mode:
        line["exchange"] = {**plan.exchange_info(), **exch_t}
        line["spmv"]["per_rank_ms"] = [[float(a), float(b)] for a, b in per_rank_all[:, :2]]
        line["spmv"]["aggregate_gflops"] = float(2 * (per_rank_all[:, 4].sum() + per_rank_all[:, 5].sum())
                                                 / ((tf + tb)) / 1e9)
    if prep is not None:
        line["preprocessing"] = prep
    if mixed is not None:
        line["mixed_canonical"] = {**mixed, "ratio_to_fp32": mixed["value"] / value}
    if multislice is not None:
        line["multislice"] = multislice
    if peer is not None:
        line["fused_peer_exchange"] = peer
    if dense is not None:
        line["dense_exchange"] = dense
    if not args.no_cpu_baseline and world == 1:
        line["cpu_baseline"] = cpu_baseline(cfg, st["nnz"], 1.0 if args.cpu_full else args.cpu_sample)
    print(json.dumps(line), flush=True)


def self_launch(args):
    """`--gpus N` (N > 1) without a torchrun environment: start N ranks of this script with
    torch.distributed.run on this node (127.0.0.1); exit non-zero if the node has fewer than N
    GPUs.  Returns the launcher's exit code."""
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus and args.transport != "host":
        print(f"bench.py: --gpus {args.gpus} needs {args.gpus} CUDA devices, this node has {have}",
              file=sys.stderr, flush=True)
        return 2
    port = os.environ.get("MASTER_PORT", str(29400 + os.getpid() % 500))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", port, os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    args = parse()
    if args.variant:
        variant_child(args)
        return
    if "WORLD_SIZE" not in os.environ and args.gpus > 1 and args.impl == "ours":
        sys.exit(self_launch(args))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if args.impl == "ours" and world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr, flush=True)
        sys.exit(2)
    if world == 1 and args.distributed and args.impl == "ours":
        for k, v in (("MASTER_ADDR", "127.0.0.1"), ("MASTER_PORT", "29533"), ("RANK", "0"),
                     ("WORLD_SIZE", "1"), ("LOCAL_RANK", "0")):
            os.environ.setdefault(k, v)
    if world > 1 or (args.distributed and args.impl == "ours"):
        import torch.distributed as dist
        if args.impl == "ours" and args.transport == "nccl":
            import torch
            torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", 0)))
            dist.init_process_group("nccl")
        else:
            dist.init_process_group("gloo")
    try:
        if args.impl == "reference":
            run_reference(args, rank, world)
        else:
            run_ours(args, rank, world)
    finally:
        if world > 1 or (args.distributed and args.impl == "ours"):
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
