#!/usr/bin/env python
"""Cold-start benchmark (BASELINE.json metric: cold-start BERT-Base/Large inference latency ms
at 1/2/4/8 GPUs).

One step = one cold-start inference of the whole hot path: the model's weights start in the
library's pinned host arena and are NOT resident on the GPU; the step runs the DeepPlan
plan (Algorithm 1 DHA selection; PT over the other ranks' PCIe links when N > 1) through
dp_infer_cold -- DMA + NCCL gather + event-gated kernels -- and ends when last_hidden_state
and the pooler output are in HBM.  Between steps the model is evicted (outside the timed
region) and L2 is flushed (a 256 MiB write).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--model bert_base] [--seq 128]
  python bench.py --impl reference ...   # the fp64 CPU oracle, timed on the host cores

Multi-GPU: one process per GPU under torch.distributed.run; rank 0 is the primary.  The
timed region is bracketed by a barrier + cuda synchronize on both sides; the value is the
max over ranks of the device-timed mean step latency.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "cold-start BERT-Base/Large inference latency ms at 1/2/4/8 GPUs; p99 serving"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--model", default="bert_base")
    ap.add_argument("--seq", type=int, default=128)
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--dtype", default="fp16", choices=["fp16", "bf16", "fp32"],
                    help="weight storage dtype (fp32 = the paper's precision, P:99; CUDA-core kernels)")
    ap.add_argument("--mode", default=None, help="plan mode (default DHA at N=1, PT_DHA at N>1)")
    ap.add_argument("--chunk-mb", type=float, default=32.0)
    ap.add_argument("--tail-mb", type=float, default=2.0)
    ap.add_argument("--h2d-streams", type=int, default=1)
    ap.add_argument("--no-graph", action="store_true", help="eager enqueue instead of CUDA-graph replay")
    ap.add_argument("--no-pdl", action="store_true")
    ap.add_argument("--profile-iters", type=int, default=10)
    ap.add_argument("--pt-transport", default="ce", choices=["dma", "sm", "ce"],
                    help="PT slots at N>1: dma = copy engine into a staging ring + NCCL send/recv (the paper's "
                         "two hops); sm = SURVEY f4 forwarder kernel (host -> primary HBM over CUDA IPC); "
                         "ce = one copy-engine DMA per piece straight into the primary's slot (CUDA IPC)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--quick", action="store_true", help="skip the other modes and per-kernel rooflines (sweeps)")
    return ap.parse_args()


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


class PcieSampler:
    """Per-GPU PCIe receive throughput from NVML (nvmlDeviceGetPcieThroughput, RX, a 20 ms
    window per sample) while the bench repeats cold starts: evidence of which GPU's link
    carried bytes (each PT secondary's link must carry its slot)."""

    def __init__(self, index: int, period_s: float = 0.02):
        self.index, self.period = index, period_s
        self.samples, self.stop_ev, self.th, self.err = [], threading.Event(), None, None

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
        except Exception as e:  # pragma: no cover (no NVML)
            self.err = f"nvml unavailable: {type(e).__name__}"
            return

        def run():
            while not self.stop_ev.is_set():
                try:
                    kbs = pynvml.nvmlDeviceGetPcieThroughput(h, pynvml.NVML_PCIE_UTIL_RX_BYTES)
                    self.samples.append(kbs * 1e3 / 1e9)  # KB/s -> GB/s
                except Exception as e:  # pragma: no cover
                    self.err = type(e).__name__
                    return
                time.sleep(self.period)

        self.th = threading.Thread(target=run, daemon=True)
        self.th.start()

    def stop(self):
        self.stop_ev.set()
        if self.th:
            self.th.join(timeout=2)
        v = self.samples
        return {"rx_gbs_mean": round(float(np.mean(v)), 2) if v else None,
                "rx_gbs_max": round(float(np.max(v)), 2) if v else None, "samples": len(v), "error": self.err}


# measured NVLink peer-copy rate per direction on this pool's B200s (B200_PROFILING.md; nominal 900)
NVLINK_GBS = 770.0


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        return json.load(open(p)), "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


def measure_h2d_peak(dp, torch, nbytes=256 << 20, reps=5):
    """Best-of-reps pinned host->device copy rate (GB/s), measured by the library on
    memory allocated exactly like its weight arena (dp_measure_h2d)."""
    return dp.measure_h2d(torch.cuda.current_device(), nbytes, reps)


def kernel_rooflines(dp, torch, m, T, peaks, peak_h2d, reps=50):
    """Per-kernel achieved rates, measured live with CUDA events on the launching stream:
    a sleep kernel holds the stream while the host enqueues `reps` launches, so the event
    interval is device time only.  Algorithmic bytes / flops per launch are in DESIGN.md §5."""
    import math
    H, F = m.hidden, m.ffn
    out = []

    def dev_us(fn):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(int(2e6 + reps * 40000))
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e3 / reps

    ridge = peaks["bf16_tflops_sustained"] * 1e12 / (peaks["hbm_gbs"] * 1e9)
    for name, N, K in (("gemm_tc fc1", F, H), ("gemm_tc q", H, H), ("gemm_tc fc2", H, F)):
        x = torch.randn(T, K, device="cuda").half()
        w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
        b = torch.randn(N, device="cuda").half()
        y = torch.empty(T, N, device="cuda").half()
        us = dev_us(lambda: dp.linear(x, K, w, b, None, 0, y, N, T, N, K, path=0))
        flops, byts = 2.0 * T * N * K, 2.0 * (N * K + T * K + T * N + N)
        if T < ridge:  # below the ridge the weight stream bounds it
            out.append({"kernel": f"{name} [{T}x{N}x{K}]", "bound": "hbm", "us": round(us, 2),
                        "achieved": round(byts / us / 1e3, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                        "frac": round(byts / us / 1e3 / peaks["hbm_gbs"], 4)})
        else:
            out.append({"kernel": f"{name} [{T}x{N}x{K}]", "bound": "tensor", "us": round(us, 2),
                        "achieved": round(flops / us / 1e6, 1), "peak": peaks["bf16_tflops_sustained"],
                        "unit": "TFLOP/s", "frac": round(flops / us / 1e6 / peaks["bf16_tflops_sustained"], 4)})
    # DHA skinny linear (weights read over PCIe exactly once)
    x = torch.randn(T, H, device="cuda").half()
    wh = dp.host_alloc(H * H * 2)
    y = torch.empty(T, H, device="cuda").half()
    us = dev_us(lambda: dp.linear(x, H, wh, None, None, 0, y, H, T, H, H, path=1))
    out.append({"kernel": f"skinny_linear DHA [{T}x{H}x{H}]", "bound": "pcie", "us": round(us, 2),
                "achieved": round(H * H * 2 / us / 1e3, 1), "peak": round(peak_h2d, 1), "unit": "GB/s",
                "frac": round(H * H * 2 / us / 1e3 / peak_h2d, 4)})
    dp.host_free(wh)
    return out


def forward_flops(m, batch, seq):
    """Algorithmic FLOPs of one forward: 2 x tokens x (linear weights) + the attention
    S^2 terms (halved for causal GPT-2)."""
    H, F, L = m.hidden, m.ffn, m.layers
    lin = L * (4 * H * H + 2 * H * F)
    att = 4.0 * seq * seq * H * L * batch * (0.5 if m.family == "gpt2" else 1.0)
    pool = 2.0 * batch * H * H if m.family != "gpt2" else 0.0
    return 2.0 * batch * seq * lin + att + pool


def cpu_baselines(m, w, ids, dtype, budget_s=10.0):
    """The CPU baselines of SURVEY §8(d), timed on this host's cores (weights already in host DRAM,
    so the CPU has no transfer): the numpy fp32 forward with the BLAS pool at all cores and at 1
    thread, and the fp64 oracle as it stands at all cores -- each the median of up to 10 runs
    after 2 warm-ups, fewer when one run is long (bounded sample).  Also returns the fp64 oracle's
    output, against which the bench checks its own last timed output."""
    from threadpoolctl import threadpool_info, threadpool_limits

    from oracle import forward as F

    def timed(compute, threads):
        with threadpool_limits(limits=threads):
            used = max([p.get("num_threads", 1) for p in threadpool_info()] or [1])
            out = None
            t0 = time.perf_counter()
            for _ in range(2):
                out = F.forward(m, w, ids, dtype, compute=compute)
            one = (time.perf_counter() - t0) / 2
            runs = max(3, min(10, int(budget_s / max(one, 1e-3))))
            ts = []
            for _ in range(runs):
                t = time.perf_counter()
                F.forward(m, w, ids, dtype, compute=compute)
                ts.append(time.perf_counter() - t)
        return float(np.median(ts) * 1e3), runs, used, out

    ncores = os.cpu_count()
    f32_all, r1, c_all, _ = timed("f32", ncores)
    f32_one, r2, _, _ = timed("f32", 1)
    f64_all, r3, _, ref = timed("f64", ncores)
    return {"fp32_all_cores_ms": round(f32_all, 3), "fp32_all_cores_runs": r1, "threads_all": c_all,
            "fp32_1_thread_ms": round(f32_one, 3), "fp32_1_thread_runs": r2,
            "fp64_oracle_all_cores_ms": round(f64_all, 3), "fp64_oracle_runs": r3}, ref


def run_reference(a):
    """--impl reference: the CPU oracle on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import synth
    m = synth.SHAPES[a.model]
    w = synth.make_weights(m, seed=0, dtype="fp16")
    ids = synth.make_ids(m, a.batch, a.seq, seed=1)
    from oracle import forward as F
    for _ in range(a.warmup):
        F.forward(m, w, ids, "fp16")
    ts = []
    steps = a.steps  # every step is one full forward of the workload (BERT-Base: ~0.3 s on 16 cores)
    for _ in range(steps):
        t = time.perf_counter()
        F.forward(m, w, ids, "fp16")
        ts.append((time.perf_counter() - t) * 1e3)
    v = float(np.mean(ts))
    cores = os.cpu_count()
    line = {"metric": METRIC, "value": round(v, 4), "unit": "ms", "n_gpus": a.gpus, "steps": steps,
            "warmup": a.warmup, "ms_per_step": round(v, 4), "higher_is_better": False, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded random-init weights, paper recipe)",
            "impl": "reference",
            "config": {"workload": f"{a.model} fp16 batch {a.batch} seq {a.seq} cold start -- reference arm: the "
                                   f"oracle's full fp64 forward on the host CPU (weights already in host DRAM, "
                                   f"fp16-rounded)",
                       "model": a.model, "global_batch": a.batch, "seq_len": a.seq, "parallelism": "host"},
            "cpu_baseline": {"value": round(v, 4), "unit": "ms", "cores": cores, "kind": "oracle",
                             "sample": f"{steps} full forwards (fp64 numpy, BLAS threads = {cores})"},
            "e2e": {"value": round(v, 4), "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def maybe_spawn(a):
    """`python bench.py --gpus N` (N > 1) without a torch.distributed launcher: re-launch this
    script under torch.distributed.run with N ranks (one process per GPU, rendezvous on
    127.0.0.1) and exit with its status; rank 0's JSON line reaches stdout unchanged."""
    if a.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def main():
    a = parse()
    maybe_spawn(a)
    if a.impl == "reference":
        run_reference(a)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_eurosys_jeongba23_b200 as dp
    import synth
    from oracle import units as OU  # noqa: F401  (byte accounting cross-check only)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # DP_BENCH_ONE_GPU=1 (tests only): every rank on device 0 and a gloo process group -- the
    # N > 1 control flow with the IPC transports (sm / ce) on a one-GPU box; NCCL refuses two
    # ranks on one device, so --pt-transport dma is not available there
    one_gpu = os.environ.get("DP_BENCH_ONE_GPU") == "1"
    if one_gpu:
        local = 0
        assert a.pt_transport != "dma" or world == 1, "DP_BENCH_ONE_GPU needs --pt-transport sm or ce"
    assert world == a.gpus, f"--gpus {a.gpus} but WORLD_SIZE {world}"
    torch.cuda.set_device(local)
    dist_on = world > 1
    if dist_on:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    red_dev = "cpu" if one_gpu else "cuda"  # gloo reduces host tensors

    m = synth.SHAPES[a.model]
    dtype = a.dtype
    w = synth.make_weights(m, seed=0, dtype=dtype)
    ids_np = synth.make_ids(m, a.batch, a.seq, seed=1)
    ctx = dp.Context([local])
    ctx.set_opts(chunk_bytes=int(a.chunk_mb * (1 << 20)), n_h2d_streams=a.h2d_streams,
                 tail_bytes=int(a.tail_mb * (1 << 20)),
                 use_graph=0 if (a.no_graph or (world > 1 and a.pt_transport == "dma")) else 1,
                 use_pdl=0 if a.no_pdl else 1, pt_transport=a.pt_transport)
    model = dp.Model(ctx, m, w, dtype)
    if dist_on and a.pt_transport == "dma":
        uid = dp.peer_unique_id() if rank == 0 else None
        box = [uid]
        dist.broadcast_object_list(box, src=0)
        ctx.peer_init(box[0], rank, world)
    elif dist_on:  # single-hop transports: CUDA IPC handles of the slots + mailboxes, no NCCL
        ctx.peer_init_ipc(rank, world)
        blocks = [None] * world
        dist.all_gather_object(blocks, model.ipc_export())
        model.ipc_import(blocks)

    # roofline denominator: pinned H2D bandwidth of this GPU's link, measured now with the
    # library's own pinned+mapped allocation (256 MiB, best of 5, CUDA events)
    peak_h2d = measure_h2d_peak(dp, torch)
    # each rank's link alone, then all k links at once (a shared PCIe switch or root complex
    # shows up as a concurrent rate below the solo one, P:148 / Table 2)
    solo = [peak_h2d]
    conc = [peak_h2d]
    if dist_on:
        solo = [None] * world
        dist.all_gather_object(solo, peak_h2d)
        torch.cuda.synchronize()
        dist.barrier()
        mine = dp.measure_h2d(local, 256 << 20, 10)
        conc = [None] * world
        dist.all_gather_object(conc, mine)
    links_info = {"h2d_solo_gbs": [round(x, 2) for x in solo], "h2d_concurrent_gbs": [round(x, 2) for x in conc],
                  "h2d_aggregate_gbs": round(float(sum(conc)), 2), "nvlink_gbs": NVLINK_GBS if world > 1 else None,
                  "nvlink_source": "B200_PROFILING.md measured peer copy per direction" if world > 1 else None}
    if dist_on:
        # pairwise concurrency matrix (rank i's rate while rank j copies) -> which rank carries
        # which PT slot (dp_select_secondaries, R25), instead of (primary + s) mod N
        pair = np.array([[s_ for s_ in solo] for _ in range(world)], dtype=np.float64)
        for i in range(world):
            for j in range(i + 1, world):
                torch.cuda.synchronize()
                dist.barrier()
                r_ = dp.measure_h2d(local, 64 << 20, 4) if rank in (i, j) else 0.0
                got = [None] * world
                dist.all_gather_object(got, r_)
                pair[i][j], pair[j][i] = got[i], got[j]
        numa = [None] * world
        dist.all_gather_object(numa, dp.device_numa_node(local))
        sec = dp.select_secondaries(solo, pair, 0, world, numa) if rank == 0 else None
        box = [sec]
        dist.broadcast_object_list(box, src=0)
        sec = box[0]
        ctx.set_slot_ranks(0, sec)
        links_info.update({"pair_gbs": [[round(x, 2) for x in row] for row in pair], "numa_node": numa,
                           "slot_ranks": sec})

    # profile on the primary, plan, share the plan (the plan never names GPUs)
    # default plan: Algorithm 1 on the link-aware model (R19); the paper's own
    # Algorithm-1 plan ("DHA") and the other engine options are timed beside it below
    mode = a.mode or ("PT_DHA_LINK_STRIPE" if world > 1 else "DHA_LINK")
    if rank == 0:
        cost = model.profile(local, a.batch, a.seq, a.profile_iters)
    else:
        cost = None
    if dist_on:
        box = [cost]
        dist.broadcast_object_list(box, src=0)
        cost = box[0]
    plan = dp.plan_generate(cost, mode, world)
    pred_ns, _, link = dp.plan_simulate(cost, plan)

    T = a.batch * a.seq
    H = m.hidden
    stream = torch.cuda.Stream()
    ids = torch.from_numpy(ids_np).cuda()
    tdt = {"fp16": torch.float16, "bf16": torch.bfloat16, "fp32": torch.float32}[dtype]
    out = torch.empty(T, H, dtype=tdt, device="cuda")
    pooled = torch.empty(a.batch, H, dtype=tdt, device="cuda") if m.family != "gpt2" else None
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(a.steps)]
    ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(a.steps)]

    def step(i=None, timed=False):
        model.evict(local) if model.is_resident(local) else None
        flush.fill_(i or 0)  # L2 flush (outside the timed region)
        torch.cuda.synchronize()
        with torch.cuda.stream(stream):
            if timed:
                ev0[i].record(stream)
            if rank == 0:
                st = model.infer_cold(plan, 0, ids, out, pooled, stream=stream)
            else:
                st = model.infer_cold_raw(plan, 0, None, a.batch, a.seq, None, None, stream.cuda_stream)
            if timed:
                ev1[i].record(stream)
        return st

    def sync_all():
        torch.cuda.synchronize()
        if dist_on:
            dist.barrier()
            torch.cuda.synchronize()

    # clocks are sampled (100 ms period) from before the warm-up to the end of the timed
    # region; the region itself is short, so it is padded to >= 1 s of repeated steps
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    for _ in range(max(3, a.warmup)):
        step()
        sync_all()
    # timed region
    sync_all()
    stats = None
    t_start = time.perf_counter()
    for i in range(a.steps):
        stats = step(i, timed=True)
        # secondaries must finish before the next eviction; the primary waits on its stream
        torch.cuda.synchronize()
        if dist_on:
            dist.barrier()
    sync_all()
    last_out = out.clone() if rank == 0 else None  # checked against the oracle below
    last_pool = pooled.clone() if (rank == 0 and pooled is not None) else None
    pad_s = 0.0 if os.environ.get("DP_BENCH_UNDER_NCU") else 1.0
    pcie = PcieSampler(local)
    pcie.start()
    while True:  # keep the GPU busy for the clock samples; rank 0 decides for every rank so
        # all ranks run the same number of cold starts (each k > 1 one is a rendezvous)
        go_on = torch.tensor([1 if time.perf_counter() - t_start < pad_s else 0], device=red_dev)
        if dist_on:
            dist.broadcast(go_on, src=0)
        if not int(go_on.item()):
            break
        step()
        sync_all()
    ck = clocks.stop()
    pcie_mine = pcie.stop()
    pcie_mine.update({"rank": rank, "device": local, "pad_steps_s": round(time.perf_counter() - t_start, 3)})
    pcie_all = [pcie_mine]
    if dist_on:
        pcie_all = [None] * world
        dist.all_gather_object(pcie_all, pcie_mine)
    lat = [ev0[i].elapsed_time(ev1[i]) for i in range(a.steps)]
    my_ms = float(np.mean(lat))
    t = torch.tensor([my_ms], dtype=torch.float64, device=red_dev)
    if dist_on:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())

    # ---- e2e: host buffers through the public API (H2D ids + D2H outputs inside) ----
    e2e_ms = None
    h2d_b = ids_np.nbytes
    d2h_b = out.numel() * out.element_size() + (pooled.numel() * pooled.element_size() if pooled is not None else 0)
    if rank == 0 or dist_on:
        ids_h = torch.from_numpy(ids_np).pin_memory()
        out_h = torch.empty(out.shape, dtype=out.dtype).pin_memory()
        pool_h = torch.empty(pooled.shape, dtype=pooled.dtype).pin_memory() if pooled is not None else None
        e2e = []
        for i in range(min(a.steps, 10)):
            model.evict(local) if model.is_resident(local) else None
            flush.fill_(1)
            sync_all()
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(stream):
                s0.record(stream)
                if rank == 0:
                    ids.copy_(ids_h, non_blocking=True)
                    model.infer_cold(plan, 0, ids, out, pooled, stream=stream)
                    out_h.copy_(out, non_blocking=True)
                    if pool_h is not None:
                        pool_h.copy_(pooled, non_blocking=True)
                else:
                    model.infer_cold_raw(plan, 0, None, a.batch, a.seq, None, None, stream.cuda_stream)
                s1.record(stream)
            stream.synchronize()
            e2e.append(s0.elapsed_time(s1))
            if dist_on:
                dist.barrier()
        t = torch.tensor([float(np.mean(e2e))], dtype=torch.float64, device=red_dev)
        if dist_on:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())

    if rank != 0:
        if dist_on:
            dist.destroy_process_group()
        return

    # warm latency (the compute-only term of the north-star roofline).  The secondaries have
    # left, so at N > 1 the model is made resident by a local cold start with the SAME method
    # vector (same DHA set, every loaded unit over this GPU's own link, k = 1)
    model.evict(local) if model.is_resident(local) else None
    plan_local = plan if world == 1 else dp._lib.PlanArrays(len(plan.method), plan.method, None, plan.s.mode, 1)
    model.infer_cold(plan_local, 0, ids, out, pooled, stream=stream)
    torch.cuda.synchronize()
    wl = []
    for i in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            e0.record(stream)
            wst = model.infer_warm(local, ids, out, pooled, stream=stream)
            e1.record(stream)
        torch.cuda.synchronize()
        wl.append(e0.elapsed_time(e1))
    warm_ms = float(np.median(wl))
    model.evict(local)

    # the same cold start under the paper's other engine options (single GPU only), for the
    # paper's comparisons (e.g. PT+DHA / DHA vs PipeSwitch)
    other_modes = {}
    if world == 1 and not os.environ.get("DP_BENCH_UNDER_NCU") and not a.quick:
        for om in ("DHA", "GREEDY", "PIPESWITCH", "BASELINE"):
            if om == mode:
                continue
            p2 = dp.plan_generate(cost, om, 1)
            ts = []
            for i in range(12):
                model.evict(local) if model.is_resident(local) else None
                flush.fill_(i)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(stream):
                    e0.record(stream)
                    model.infer_cold(p2, 0, ids, out, pooled, stream=stream)
                    e1.record(stream)
                torch.cuda.synchronize()
                if i >= 2:
                    ts.append(e0.elapsed_time(e1))
            model.evict(local)
            other_modes[om] = {"ms": round(float(np.mean(ts)), 4), "dha_units": int(p2.method.sum()),
                               "predicted_ms": round(dp.plan_simulate(cost, p2)[0] / 1e6, 4)}

    # bytes per host link come from the plan (the simulator's link_bytes equal the bytes each
    # link's DMAs carry, bit-exactly -- tests/test_gpu_forward.py); rank 0's own stats only see
    # its own link when the partitions travel on other ranks
    link_plan = [int(b) for b in link][:world]
    h2d_bytes = int(sum(link_plan))
    assert world > 1 or h2d_bytes == int(stats["h2d_bytes"][0]), (h2d_bytes, stats["h2d_bytes"])
    dha_bytes = int(stats["dha_weight_bytes"])
    link_bytes = h2d_bytes + dha_bytes  # bytes the path must move over host links per step
    per_link = max([link_plan[0] + dha_bytes] + link_plan[1:])  # DHA reads use the primary's link
    nvl_bytes = int(sum(link_plan[1:]))  # gathered into the primary over NVLink
    achieved = link_bytes / (ms * 1e-3) / 1e9
    total_w = model.nbytes
    agg = links_info["h2d_aggregate_gbs"]
    # north star: R(k) = (weight bytes not yet resident) / (measured concurrent aggregate H2D of
    # the k links) + NVLink gather time, versus warm compute; the algorithmic variant moves only
    # the bytes the plan must move and overlaps H2D with the gather (max instead of +)
    R_lit = total_w / (agg * 1e9) * 1e3 + (nvl_bytes / (NVLINK_GBS * 1e9) * 1e3 if world > 1 else 0.0)
    R_alg = max(per_link / (min(links_info["h2d_concurrent_gbs"]) * 1e9) * 1e3,
                nvl_bytes / (NVLINK_GBS * 1e9) * 1e3 if world > 1 else 0.0)  # busiest link
    peaks, peaks_src = measured_peaks()
    fwd_flops = forward_flops(m, a.batch, a.seq)
    # compute floor of the forward: the tensor pipe for 16-bit storage; for fp32 storage the kernels
    # are CUDA-core FMA (no fp32 tcgen05 kind): 148 SMs x 128 fp32 lanes x 2 flops x 1.965 GHz
    fp32_alu_tflops = 148 * 128 * 2 * 1.965e9 / 1e12
    T_compute = fwd_flops / ((fp32_alu_tflops if dtype == "fp32" else peaks["bf16_tflops_sustained"]) * 1e12) * 1e3
    krl = None if (os.environ.get("DP_BENCH_UNDER_NCU") or a.quick) else kernel_rooflines(dp, torch, m, T, peaks,
                                                                                          peak_h2d)

    cpu = None
    check = None
    if not a.no_cpu_baseline:
        cb, (ref, ref_pool) = cpu_baselines(m, w, ids_np, dtype)
        cpu = {"value": cb["fp32_all_cores_ms"], "unit": "ms", "cores": cb["threads_all"], "kind": "oracle",
               "sample": f"median of {cb['fp32_all_cores_runs']} full {a.model} forwards (batch {a.batch}, seq "
                         f"{a.seq}) after 2 warm-ups, numpy fp32 (oracle.forward compute='f32'), BLAS threads = "
                         f"{cb['threads_all']}; weights already in host DRAM (no transfer)", **cb}
        # the bench's own last timed output against the fp64 oracle on the same inputs (north star:
        # max-abs <= 1e-2 for fp16; <= 1e-4 relative for fp32 (R24); bf16: 1e-2 + the
        # representation error of bf16 activations (R15), from the oracle's act_round variant)
        got = last_out.float().cpu().numpy().astype(np.float64).reshape(ref.shape)
        err = float(np.abs(got - ref).max())
        rel = float((np.abs(got - ref) / np.maximum(1.0, np.abs(ref))).max())
        if dtype == "fp32":
            tol, ok = 1e-4, rel <= 1e-4
        else:
            rep = 0.0
            if dtype == "bf16":
                from oracle import forward as F
                rep = float(np.abs(F.forward(m, w, ids_np, dtype, act_round=dtype)[0] - ref).max())
            tol = 1e-2 + rep
            ok = err <= tol
        check = {"vs": "fp64 oracle forward of the same weights and ids", "max_abs_err": err, "max_rel_err": rel,
                 "tol": tol, "tol_kind": "relative" if dtype == "fp32" else "max-abs", "ok": bool(ok)}
        if last_pool is not None:
            perr = float(np.abs(last_pool.float().cpu().numpy().astype(np.float64) - ref_pool).max())
            prel = float((np.abs(last_pool.float().cpu().numpy().astype(np.float64) - ref_pool) /
                          np.maximum(1.0, np.abs(ref_pool))).max())
            check["max_abs_err_pooler"] = perr
            check["ok"] = bool(check["ok"] and ((prel <= 1e-4) if dtype == "fp32" else (perr <= tol)))
        if not check["ok"]:
            print(f"bench: OUTPUT CHECK FAILED {check}", file=sys.stderr, flush=True)

    line = {
        "metric": METRIC, "value": round(ms, 4), "unit": "ms", "n_gpus": world, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": round(ms, 4), "higher_is_better": False, "scaling": "strong",
        "vs_baseline": None, "dtype": dtype, "data": "synthetic (seeded random-init weights of the HF shapes)",
        "config": {"workload": f"{a.model} {dtype} batch {a.batch} seq {a.seq} cold start from pinned host memory, "
                               f"plan {mode} k={world}",
                   "model": a.model, "global_batch": a.batch, "seq_len": a.seq, "parallelism": f"pt{world}",
                   "plan_mode": mode, "dha_units": int(plan.method.sum()), "units": int(len(plan.method)),
                   "chunk_bytes": int(a.chunk_mb * (1 << 20)), "h2d_streams": a.h2d_streams,
                   "pt_transport": a.pt_transport if world > 1 else None,
                   "l2": "flushed between steps (256 MiB write)"},
        "roofline": {"bound": "pcie", "achieved": round(achieved, 2), "peak": round(agg, 2), "unit": "GB/s",
                     "frac": round(achieved / agg, 4), "traffic": None,
                     "bytes_per_step": link_bytes,
                     "peak_source": "pinned 256 MiB H2D measured in this run (k links at once when k > 1)",
                     "note": "dominant component is the host-link transfer (copy engine + DHA reads); "
                             "ncu cannot see copy-engine traffic"},
        "other_modes": other_modes,
        "speedup_vs_pipeswitch": (round(other_modes["PIPESWITCH"]["ms"] / ms, 3)
                                  if "PIPESWITCH" in other_modes else None),
        "path_roofline": {"R_literal_ms": round(R_lit, 4), "R_algorithmic_ms": round(R_alg, 4),
                          "T_warm_ms": round(warm_ms, 4), "T_compute_floor_ms": round(T_compute, 4),
                          "forward_gflop": round(fwd_flops / 1e9, 2), "nvlink_bytes": nvl_bytes,
                          # the bound is never raised by our own warm forward: transfer vs the
                          # forward's FLOPs at the sustained tensor peak
                          "bound_ms": round(max(R_lit, T_compute), 4),
                          "value_over_bound": round(ms / max(R_lit, T_compute), 4),
                          "value_over_R_literal_or_warm": round(ms / max(R_lit, warm_ms), 4),
                          "value_over_R_algorithmic": round(ms / max(R_alg, T_compute), 4),
                          "predicted_ms": round(pred_ns / 1e6, 4)},
        "clocks": ck,
        "e2e": {"value": round(e2e_ms, 4) if e2e_ms else None, "unit": "ms", "h2d_bytes_per_step": int(h2d_b),
                "d2h_bytes_per_step": int(d2h_b)},
        "gpu_launches": int(stats["n_kernels"]) * a.steps,
        "stats": {"h2d_bytes": h2d_bytes, "dha_weight_bytes": dha_bytes, "copies": stats["n_copies"],
                  "events": stats["n_events"], "kernels_per_step": stats["n_kernels"],
                  "enqueue_us": round(stats["wall_enqueue_us"], 1), "step_ms_min": round(min(lat), 4),
                  "step_ms_max": round(max(lat), 4), "warm_kernels": wst["n_kernels"]},
        "peaks": {"source": peaks_src, "hbm_gbs": peaks.get("hbm_gbs"),
                  "bf16_tflops_sustained": peaks.get("bf16_tflops_sustained")},
        "kernel_rooflines": krl,
        "cpu_baseline": cpu,
        "check": check,
        "pcie_rx": pcie_all,
        "links": links_info,
    }
    print(json.dumps(line), flush=True)
    model.close()
    ctx.close()
    if dist_on:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
