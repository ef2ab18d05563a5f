"""bench.py -- ConcatBatch encoder forward throughput on B200 (non-pad tokens/s).

Contract (driver): ``python bench.py --gpus N --steps K --warmup W [--impl reference]``;
for N > 1 launched under torchrun, one rank per GPU.  Prints ONE JSON line on rank 0.

A step = one pass of the whole hot path -- pack_embed -> S x [QKV GEMM -> segment-masked
attention -> W_O GEMM + residual -> LN -> FFN1 + act -> FFN2 + residual -> LN] -> unpack --
over one packed batch of B rows x L slots per GPU (BASELINE.json configs[1]: Transformer-
base, L = 128, ParaCrawl-like lengths, bf16, B = 256 rows per GPU).  Weak scaling: each
rank packs its own seeded request stream (seed + 1000 * rank); weights are generated on
rank 0 and broadcast once (NCCL); there is no per-step collective.

value: device time (CUDA events on the launching stream), inputs resident in HBM, the
       forward replayed from a CUDA graph, L2 flushed (256 MiB write) between steps,
       max over ranks; value = sum of non-pad tokens over ranks / max time.
e2e:   the same metric through the C ABI with HOST buffers: per step tcb_pack (C++) and
       tcb_session_run (the library uploads the segment table + pinned token ids, runs forward +
       unpack, downloads the per-request outputs [T, d] into pinned host memory on a copy
       stream), tcb_session_wait, the host reads the outputs; two slots (the download of step i
       overlaps step i+1); host wall clock.
roofline: the dominant kernel class (largest device time per step), each launch timed by CUDA
       event nodes inside a graph-replayed step (tcb_profile_*; L2 flushed per replay);
       algorithmic flops / bytes per class in DESIGN.md section 7 (GEMMs: 2 T d_in d_out per
       layer over non-pad tokens T) against the burst bf16 peak / hbm_gbs of
       MEASURED_PEAKS.json; every class is listed under roofline.classes.
cpu_baseline / --impl reference: the float64 oracle (oracle/, test infrastructure) on a
       bounded sample of the same workload, on this host's cores.
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

import tcb_workload as wl  # noqa: E402

METRIC = "non-pad tokens/s, ConcatBatch encoder fwd at 1/2/4/8 B200; % TC peak"
UNIT = "tokens/s"


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """SM clocks / throttle reasons sampled DURING the timed region: NVML every 2 ms
    (nvidia_ml_py), else nvidia-smi every 0.2 s."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []          # (sm_mhz, max_mhz, power_w, set(reasons))
        self.source = None
        self._stop = threading.Event()
        self._t = None
        self._nvml = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nvml = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(gpu)
            self._max = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
            self.source = "nvml"
        except Exception:
            self._nvml = None

    def _sample_nvml(self):
        nv = self._nvml
        sm = nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM)
        try:
            pw = nv.nvmlDeviceGetPowerUsage(self._h) / 1000.0
        except Exception:
            pw = None
        bits = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
        masks = [0x8, 0x40, 0x20, 0x4]   # hw_slowdown, hw_thermal, sw_thermal, sw_power_cap
        reasons = {n for n, m in zip(self.NAMES, masks) if bits & m}
        self.rows.append((float(sm), float(self._max), pw, reasons))

    def _sample_smi(self):
        out = subprocess.run(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                              "--format=csv,noheader,nounits"],
                             capture_output=True, text=True, timeout=5).stdout
        for line in out.strip().splitlines():
            r = [x.strip() for x in line.split(",")]
            num = lambda x: float(x) if x.replace(".", "").isdigit() else None  # noqa: E731
            reasons = {self.NAMES[i] for i in range(4) if len(r) > 5 + i and r[5 + i].lower() == "active"}
            self.rows.append((num(r[1]), num(r[2]), num(r[3]), reasons))
        self.source = "nvidia-smi"

    def _run(self):
        while not self._stop.is_set():
            try:
                if self._nvml is not None:
                    self._sample_nvml()
                else:
                    self._sample_smi()
            except Exception:
                pass
            self._stop.wait(0.002 if self._nvml is not None else 0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["clock sampling unavailable"],
                    "samples": 0}
        sm = [r[0] for r in self.rows if r[0] is not None]
        mx = [r[1] for r in self.rows if r[1] is not None]
        pw = [r[2] for r in self.rows if r[2] is not None]
        reasons = sorted(set().union(*[r[3] for r in self.rows]))
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "power_w_max": max(pw) if pw else None, "samples": len(self.rows),
                "source": self.source}


def make_batches(key: str, rank: int, nbatches: int):
    """Seeded packed batches for this rank: (lengths, ids) filling B rows of L slots."""
    wlc = wl.WORKLOADS[key]
    out = []
    for b in range(nbatches):
        seed = wlc.seeds[0] + 1000 * rank + 97 * b
        lengths = wl.lengths_filling(wlc.lengths, wlc.rows, wlc.row_len, seed, 0.995)
        ids = wl.draw_token_ids(int(lengths.sum()), wlc.model.vocab, wlc.seeds[1] + 1000 * rank + 97 * b)
        out.append((lengths, ids))
    return out


def cpu_oracle_sample(key: str, lengths, ids, weights, budget_s: float = 12.0, max_rows=16,
                      threads: int = 0):
    """Time the f64 oracle (as it stands) row by row on this host until ~budget_s.
    threads = 0: every core of this process's affinity; 1: the single-thread baseline."""
    import oracle
    wlc = wl.WORKLOADS[key]
    model = wlc.model
    names = wl.weight_names(model)
    pk = oracle.pack(lengths, wlc.row_len, wlc.rows)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], wlc.row_len)
    seg = lay["segment_ids"]
    L = wlc.row_len
    avail = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()
    cores = oracle.set_num_threads(threads if threads > 0 else avail)
    tokens, elapsed, rows = 0, 0.0, 0
    try:
        while elapsed < budget_s and rows < min(max_rows, pk["num_rows"]):
            t0 = time.perf_counter()
            oracle.encoder_rows(model, weights, names, ids, lay, L, [rows])
            elapsed += time.perf_counter() - t0
            tokens += int(np.sum(seg[rows * L:(rows + 1) * L] >= 0))
            rows += 1
    finally:
        oracle.set_num_threads(avail)
    return {"value": tokens / elapsed, "unit": UNIT, "cores": int(cores),
            "kind": "oracle",
            "sample": f"first {rows} packed rows ({tokens} non-pad tokens) of the rank-0 batch, "
                      f"{model.name} L={L}, float64, {elapsed:.1f} s, {cores} thread(s)"}


def run_reference(args):
    """--impl reference: the f64 oracle timed as it stands, rank 0 only."""
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    if rank != 0:
        return 0
    key = args.workload
    wlc = wl.WORKLOADS[key]
    (lengths, ids), = make_batches(key, 0, 1)
    weights = wl.draw_weights(wlc.model, wlc.seeds[2])
    import oracle
    names = wl.weight_names(wlc.model)
    pk = oracle.pack(lengths, wlc.row_len, wlc.rows)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], wlc.row_len)
    L = wlc.row_len
    seg = lay["segment_ids"]
    # each step: a bounded sample (one packed row) of the workload
    def step(i):
        r = i % pk["num_rows"]
        oracle.encoder_rows(wlc.model, weights, names, ids, lay, L, [r])
        return int(np.sum(seg[r * L:(r + 1) * L] >= 0))
    for i in range(args.warmup):
        step(i)
    toks, t0 = 0, time.perf_counter()
    for i in range(args.steps):
        toks += step(args.warmup + i)
    el = time.perf_counter() - t0
    v = toks / el
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()
    line = {"metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * el / max(args.steps, 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "impl": "reference",
            "config": {"workload": wlc.name, "model": wlc.model.name, "row_len": L,
                       "rows_per_gpu": wlc.rows, "sample_per_step": "one packed row"},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": "one packed row per step of the rank-0 batch"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_online(args):
    """--online: BASELINE configs[4] -- one Poisson request stream (WMT-like lengths) over all
    ranks (paper_conf_icpp_fuc0z22_b200/serve_dist.py): a dispatcher thins it into one
    Poisson(lambda / W) substream per rank, each rank serves its share with its own scheduler
    (DAS) and encoder replica (Transformer-big encoder, 128 x 256 rows, CUDA-graph replay per
    time slot), no per-step collective.  lambda = load x W x the measured single-GPU capacity.
    value = tokens answered by all ranks / the longest rank's serving clock (scheduler host
    time + device time per slot)."""
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_fuc0z22_b200 as tcb
    from paper_conf_icpp_fuc0z22_b200 import dist as tdist
    from paper_conf_icpp_fuc0z22_b200 import serve_dist as sd

    rank, world = tdist.init("nccl")
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    wlc = wl.WORKLOADS["c5"]
    model = wlc.model
    names = wl.weight_names(model)
    weights_np = wl.draw_weights(model, wlc.seeds[2]) if rank == 0 else None
    views = tdist.broadcast_weights(model, names, weights_np, dev)
    enc = tcb.Encoder(model, None, names, device=str(dev), tensors=views)
    B, L = wlc.rows, wlc.row_len
    cap, tau = sd.capacity(enc, wlc.lengths, B, L, wlc.seeds[0])
    # every rank must draw the same global stream: agree on the capacity (max over ranks)
    t = torch.tensor([cap, tau], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    cap, tau = float(t[0]), float(t[1])
    rate = args.load * world * cap
    horizon = args.horizon
    n = int(rate * horizon * 1.1) + 1000
    sub = sd.substream(rank, world, n, rate, wlc.lengths, L, tau, wlc.seeds[0] + 17)
    # warm-up: a short run of the same serving loop (graph capture, scheduler, allocator)
    sd.serve_rank(enc, {k: v[:2000] for k, v in sub.items()}, model.vocab, B, L, "das",
                  min(horizon, 5 * tau), wlc.seeds[1] + rank)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        res = sd.serve_rank(enc, sub, model.vocab, B, L, "das", horizon, wlc.seeds[1] + rank)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    red = sd.reduce_results(res, world)
    if rank == 0:
        line = {
            "metric": "sustained non-pad tokens/s, online DAS over a Poisson stream (C5)",
            "value": red["tokens_per_s"], "unit": UNIT, "n_gpus": world,
            "steps": int(red["batches"]), "warmup": 1,
            "ms_per_step": 1e3 * red["seconds"] / max(red["batches"] / world, 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
            "data": "synthetic (Poisson arrivals, WMT-like lengths, R29 deadlines, random-init weights)",
            "config": {"workload": "c5-online", "model": model.name, "layers": model.num_layers,
                       "d_model": model.d_model, "rows_per_gpu": B, "row_len": L,
                       "policy": "das (eta = q = 1/2)", "load_x_capacity": args.load,
                       "arrival_rate_req_per_s": rate, "single_gpu_capacity_req_per_s": cap,
                       "full_batch_ms": tau * 1e3, "horizon_s": horizon,
                       "parallelism": f"dp{world} (Poisson thinning per rank, weights broadcast once)"},
            "online": red,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)        # the driver runs --steps 20 --warmup 5 (BENCH_r01.json)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c2", choices=sorted(wl.WORKLOADS))
    ap.add_argument("--rows", type=int, default=0,
                    help="batch rows per GPU (default: the workload's B; a sweep knob, not the bench line)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--online", action="store_true",
                    help="C5 online serving: one Poisson stream over all ranks (serve_dist.py)")
    ap.add_argument("--load", type=float, default=2.0, help="--online: arrival rate / capacity")
    ap.add_argument("--horizon", type=float, default=0.3, help="--online: served seconds per rank")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)
    if args.online:
        return run_online(args)

    import torch
    import torch.distributed as dist

    import paper_conf_icpp_fuc0z22_b200 as tcb
    from paper_conf_icpp_fuc0z22_b200 import dist as tdist

    rank, world = tdist.init("nccl")
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    key = args.workload
    if args.rows > 0:                     # batch-size sweep: same workload, B rows per GPU
        import dataclasses
        wl.WORKLOADS[key] = dataclasses.replace(wl.WORKLOADS[key], rows=args.rows)
    wlc = wl.WORKLOADS[key]
    model = wlc.model
    names = wl.weight_names(model)
    L, B = wlc.row_len, wlc.rows

    # weights: drawn on rank 0, one NCCL broadcast of the flat buffers
    weights_np = wl.draw_weights(model, wlc.seeds[2]) if rank == 0 else None
    views = tdist.broadcast_weights(model, names, weights_np, dev)
    enc = tcb.Encoder(model, None, names, device=str(dev), tensors=views)

    batches = make_batches(key, rank, 4)
    plans = [tcb.tcb_pack(l, L, B) for l, _ in batches]
    plan = plans[0]
    info = plan.info
    M = info["num_slots"]
    assert info["num_rows"] == B, info
    tokens_rank = info["placed_tokens"]
    d_segtab = torch.from_numpy(plan.segtab()).to(dev)
    d_ids = torch.from_numpy(batches[0][1]).to(dev)
    rows = enc.alloc_rows(M)
    out = torch.empty((info["total_tokens"], model.d_model), dtype=enc.dtype, device=dev)
    stream = torch.cuda.Stream(device=dev)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)

    # forward + unpack: tcb_encoder_forward_unpacked (the unpack fused into the last FFN2 +
    # LN2 where the L2-exchange kernel runs; TCB_BENCH_UNPACK=separate: the two calls)
    separate_unpack = os.environ.get("TCB_BENCH_UNPACK") == "separate"

    def fwd():
        if separate_unpack:
            enc.encoder_forward(plan, d_segtab, d_ids, rows, stream=stream)
            enc.unpack(plan, d_segtab, rows, out, stream=stream)
        else:
            enc.encoder_forward_unpacked(plan, d_segtab, d_ids, out, rows, stream=stream)

    # launches per step (counted from the library's own counter on one eager step)
    c0 = tcb.launch_count()
    with torch.cuda.stream(stream):
        fwd()
    stream.synchronize()
    launches_per_step = tcb.launch_count() - c0

    graph = None
    if not args.no_graph:
        with torch.cuda.stream(stream):
            fwd()
        stream.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=stream):
            fwd()

    def step():
        if graph is not None:
            graph.replay()
        else:
            fwd()

    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            step()
    stream.synchronize()

    # ---- timed region: device time, L2 flushed between steps -----------------------------
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        with torch.cuda.stream(stream):
            for i in range(args.steps):
                flush.zero_()
                ev[i][0].record(stream)
                step()
                ev[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    if os.environ.get("TCB_BENCH_DUMP_STEPS"):            # diagnostics: per-step device times
        print("step_ms " + " ".join("%.4f" % t for t in step_ms), file=sys.stderr, flush=True)
    ms = sum(step_ms)
    t_local = torch.tensor([ms, float(tokens_rank)], dtype=torch.float64, device=dev)
    if world > 1:
        tmax = t_local.clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        tsum = t_local.clone()
        dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
        ms_max, tokens_all = float(tmax[0]), float(tsum[1])
    else:
        ms_max, tokens_all = ms, float(tokens_rank)
    value = tokens_all * args.steps / (ms_max / 1e3)
    ms_per_step = ms_max / args.steps

    # ---- roofline: per-kernel-class durations inside the graph-replayed step -----------------
    # The same forward + unpack is captured once more with profiling on: every launch sits
    # between two event-record nodes of the graph, so each replay times every kernel (warm
    # caches and the pipeline's own L2 state, as in the timed step; the event nodes only remove
    # the programmatic overlap between neighbouring kernels).  L2 flushed before every replay.
    tcb.profile_enable(True)
    with torch.cuda.stream(stream):
        fwd()                                           # warm-up of the profiled path
    stream.synchronize()
    tcb.profile_collect()
    pgraph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(pgraph, stream=stream):
        fwd()
    tcb.profile_enable(False)
    prof = {}
    pstep = []
    with torch.cuda.stream(stream):
        for _ in range(args.steps):
            flush.zero_()
            pa, pb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            pa.record(stream)
            pgraph.replay()
            pb.record(stream)
            stream.synchronize()
            pstep.append(pa.elapsed_time(pb))
            for c, (t, n) in tcb.profile_snapshot().items():
                m0, n0 = prof.get(c, (0.0, 0))
                prof[c] = (m0 + t, n0 + n)
    del pgraph
    tcb.profile_collect()                               # release the records' events
    peaks, peak_src = _peaks()
    d, S, f = model.d_model, model.num_layers, model.d_ff
    T = tokens_rank
    gemm_cls = ["gemm_qkv", "gemm_o", "gemm_ffn1", "gemm_ffn2"]
    gemm_flops = 2.0 * T * S * (3 * d * d + d * d + 2 * d * f)
    attn_flops = 4.0 * d * S * info["useful_score_elems"]
    tc_burst = peaks["bf16_tflops"]
    tc_sust = peaks.get("bf16_tflops_sustained", tc_burst)
    hbm_peak = peaks["hbm_gbs"]
    esz = 2 if model.dtype == "bf16" else 4
    fused_ln = d in (512, 768, 1024) and model.dtype == "bf16"
    # algorithmic work per forward of each kernel class: flops for the
    # contractions (non-pad tokens only), bytes for the HBM-bound kernels
    work = {
        "gemm_qkv": ("tensor", 2.0 * T * S * 3 * d * d),
        "gemm_o": ("tensor", 2.0 * T * S * d * d),
        "gemm_ffn1": ("tensor", 2.0 * T * S * d * f),
        "gemm_ffn2": ("tensor", 2.0 * T * S * d * f),
        # attention is HBM-bound (AI = E[l]/2 flop/B < ridge): Q, K, V in + O
        # out per non-pad token per layer; its useful (segment-diagonal) flop rate is reported
        # next to it
        "attention": ("hbm", 1.0 * T * S * 4 * d * esz),
        "embed": ("hbm", T * (4 + 2 * d * esz + 8)),
        "layernorm": ("hbm", 0.0 if fused_ln else 2.0 * S * T * 2 * d * esz),
        "unpack": ("hbm", T * 2 * d * esz),
    }
    # the kernels that run for each class (api.cu / linear_tc.cu dispatch)
    ln_o = {512: "linear_ln_kernel<false>", 768: "linear_lnc_kernel<3>", 1024: "linear_lnc_kernel<4>"}
    ln_2 = {512: "linear_lng_kernel<2,256>", 768: "linear_lng_kernel<3,256>", 1024: "linear_lng_kernel<4,256>"}
    names = {"gemm_qkv": "linear_tc_kernel<2,256,EPI_BIAS> (QKV)",
             "gemm_o": f"{ln_o.get(d)} (W_O + residual + LN1)" if fused_ln else "linear_tc_kernel (W_O + residual)",
             "gemm_ffn1": "linear_tc_kernel<2,256,EPI_ACT> (FFN1 + act)",
             "gemm_ffn2": f"{ln_2.get(d)} (FFN2 + residual + LN2)" if fused_ln else "linear_tc_kernel (FFN2 + residual)",
             "attention": ("v3s::attn_tc3s_kernel" if L <= 128 else "v3::attn_tc3_kernel") +
                          " (segment-masked attention; Q,K,V in + O out)",
             "embed": "pack_embed_kernel", "layernorm": "layernorm_kernel", "unpack": "unpack_kernel"}
    # Per-class duration in the REAL step: the profiled replay (an event node before and after
    # every launch) gives each class's share of the step; the event nodes also serialise the
    # launches (no programmatic dependent launch across them) and expose every prologue, so
    # the profiled replay runs longer than the real step.  The headline figure apportions the
    # real (graph, PDL) step time by those shares; the isolated event-timed figure is kept
    # under "isolated".  The ncu launch list's shares agree (scripts/r02/share_check.py).
    total_prof_ms = sum(v[0] for v in prof.values()) / args.steps
    classes = {}
    for c, (bound, w) in work.items():
        ms_c, n_c = prof.get(c, (0.0, 0))
        if n_c == 0 or ms_c <= 0 or w <= 0:
            continue
        n_step = n_c / args.steps
        share = (ms_c / args.steps) / total_prof_ms
        us_in_step = 1e3 * share * ms_per_step / n_step
        us_iso = 1e3 * ms_c / n_c
        w_launch = w / n_step
        if bound == "tensor":
            ach, ach_iso, pk, unit = w_launch / us_in_step / 1e6, w_launch / us_iso / 1e6, tc_burst, "TFLOP/s"
        else:
            ach, ach_iso, pk, unit = w_launch / us_in_step / 1e3, w_launch / us_iso / 1e3, hbm_peak, "GB/s"
        classes[c] = {"kernel": names[c], "bound": bound, "achieved": ach, "peak": pk, "unit": unit,
                      "frac": ach / pk, "launches_per_step": n_step, "share_of_step": share,
                      "ms_per_step": share * ms_per_step, "us_per_launch": us_in_step,
                      "work_per_launch": w_launch,
                      "isolated": {"us_per_launch": us_iso, "achieved": ach_iso, "frac": ach_iso / pk}}
        if bound == "tensor":
            classes[c]["frac_vs_sustained"] = ach / tc_sust
        if c == "attention":
            classes[c]["useful_tflops"] = attn_flops / n_step / (us_in_step * 1e-6) / 1e12
    dom = max(classes, key=lambda c: classes[c]["ms_per_step"])
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        try:
            traffic = json.load(open(tpath)).get(key, {}).get(dom)
        except Exception:
            traffic = None
    dc = classes[dom]
    roofline = {"bound": dc["bound"], "kernel": dc["kernel"], "class": dom,
                "achieved": dc["achieved"], "peak": dc["peak"], "unit": dc["unit"],
                "frac": dc["frac"], "traffic": traffic,
                "peak_source": f"{peak_src} " + ("bf16_tflops (burst: the step runs at the clocks of a "
                                                 "short burst, see clocks)" if dc["bound"] == "tensor" else "hbm_gbs"),
                "timing": "algorithmic work per launch / the kernel's average duration in the timed "
                          "(graph-replayed, L2-flushed) step = its share of the step (CUDA events recorded "
                          "as event nodes around every launch of a profiled replay) x the step time / "
                          "launches; the event-isolated duration is under classes[...].isolated",
                "work_per_launch": dc["work_per_launch"],
                "us_per_launch": dc["us_per_launch"],
                "share_of_step": dc["share_of_step"],
                "isolated": dc["isolated"],
                "profiled_graph_ms_per_step": float(np.median(pstep)),
                "sum_of_kernels_ms_per_step": total_prof_ms,
                "gemm_class_frac": (gemm_flops / (sum(classes[c]["ms_per_step"] for c in gemm_cls if c in classes)
                                                  / 1e3) / 1e12) / tc_burst,
                "classes": classes}
    whole_tc = (gemm_flops + attn_flops) / (ms_per_step / 1e3) / 1e12

    # ---- e2e: the C-ABI host-buffer path (tcb_session_run), every step ---------------------
    # Per step: tcb_pack (host C++) -> tcb_session_run(plan, pinned host ids, pinned host out):
    # the library uploads the segment table and the ids, runs forward + unpack and copies the
    # [T, d] outputs back -- on a copy stream, so step i's download overlaps step i+1 (two
    # slots) -- and the host reads each step's outputs once tcb_session_wait returns.
    pinned_ids = [torch.from_numpy(i).pin_memory() for _, i in batches]
    max_t = max(p.info["total_tokens"] for p in plans)
    out_host = [torch.empty((max_t, model.d_model), dtype=enc.dtype).pin_memory() for _ in range(2)]
    sess = enc.session(B, L, max_t)
    cstream = torch.cuda.Stream(device=dev)
    tickets, pending = [None, None], [0, 0]
    h2d = d2h = 0
    checksum = 0.0

    def consume(k):
        nonlocal checksum
        if tickets[k] is not None:
            sess.wait(tickets[k])                              # step's outputs are on the host
            checksum += float(out_host[k][pending[k] - 1, 0])
            tickets[k] = None

    def e2e_step(i):
        nonlocal h2d, d2h
        k = i & 1
        lengths, ids = batches[i % len(batches)]
        p = tcb.tcb_pack(lengths, L, B)                         # host packer (C++)
        consume(k)                                              # output slot k is free again
        T = p.info["total_tokens"]
        tickets[k] = sess.run(p, pinned_ids[i % len(batches)], out_host[k], stream, cstream)
        pending[k] = T
        h2d += int(lib_words(p)) * 4 + len(ids) * 4
        d2h += T * model.d_model * out_host[k].element_size()

    def lib_words(p):
        return tcb._lib.lib().tcb_plan_segtab_words(p.handle)

    def drain():
        consume(0)
        consume(1)
        torch.cuda.synchronize(dev)

    for i in range(args.warmup):
        e2e_step(i)
    drain()
    h2d = d2h = 0
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for i in range(args.steps):
        e2e_step(i)
    drain()
    e2e_s = time.perf_counter() - t0
    e2e_t = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_tokens = sum(plans[i % len(plans)].info["placed_tokens"] for i in range(args.steps))
    e2e_value = e2e_tokens * world / float(e2e_t[0])
    del sess

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        w64 = wl.draw_weights(model, wlc.seeds[2])
        cpu = cpu_oracle_sample(key, batches[0][0], batches[0][1], w64)
        # the same oracle on ONE host thread (SURVEY 8(d) / BASELINE.md: next to the all-core run)
        cpu["single_thread"] = cpu_oracle_sample(key, batches[0][0], batches[0][1], w64,
                                                 budget_s=8.0, max_rows=4, threads=1)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
            "data": "synthetic (seeded ParaCrawl-like lengths, random-init weights)",
            "config": {"workload": wlc.name, "model": model.name, "layers": S, "d_model": d,
                       "heads": model.num_heads, "d_ff": model.d_ff, "row_len": L,
                       "rows_per_gpu": B, "global_batch_rows": B * world,
                       "non_pad_tokens_per_gpu": tokens_rank,
                       "padding_fraction": 1.0 - tokens_rank / M,
                       "attention_tiles_skipped_128": 1.0 - info["kv_tiles_visited"] / info["kv_tiles_dense"]
                       if info["kv_tiles_dense"] > 0 else None,
                       "attention_score_elems_executed_vs_dense": info["executed_score_elems"] / (B * L * L),
                       "attention_useful_fraction_of_executed": info["useful_score_elems"] / max(info["executed_score_elems"], 1),
                       "parallelism": f"dp{world} (rows sharded, weights broadcast once)",
                       "l2": "flushed (256 MiB write) between timed steps",
                       "cuda_graph": graph is not None},
            "ms_per_step_p10_p50_p90": [float(np.percentile(step_ms, q)) for q in (10, 50, 90)],
            "tc_frac_whole_step": whole_tc / tc_burst,
            "tc_frac_whole_step_vs_sustained": whole_tc / tc_sust,
            "tc_whole_step_tflops": whole_tc,
            "gpu_launches": int(launches_per_step * args.steps),
            "roofline": roofline,
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": h2d // args.steps,
                    "d2h_bytes_per_step": d2h // args.steps,
                    "path": "tcb_pack + tcb_session_run (C ABI, host buffers: pinned ids in, pinned [T, d] out; the library uploads the segment table + ids, runs tcb_encoder_forward_unpacked (unpack fused into the last FFN2 + LN2), downloads on a copy stream) + tcb_session_wait, host reads each step's outputs; two slots (step i's download overlaps step i+1)"},
            "clocks": clk.summary(),
            "cpu_baseline": cpu,
            "paper_context": "paper reports only end-to-end serving on 1x V100 (<~4e3 tok/s incl. decoder); no encoder tokens/s",
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
