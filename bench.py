#!/usr/bin/env python
"""Throughput of the Mimose checkpointed training step under a fixed memory
budget with a dynamic sequence length (BASELINE.json metric), on N GPUs.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config bert-base]
    python bench.py --impl reference ...      # the fp64 CPU oracle arm

One step = Mimose plan lookup (estimator + Algorithm 1 on a cache miss)
+ forward + backward with recompute + AdamW, on one synthetic SWAG-like batch
(DESIGN "Input recipe").  The sheltered phase (collect_iters shuttled
iterations) runs before the warm-up and is reported separately.
Multi-GPU: one process per GPU (torchrun), weak scaling, the same S_t on every
rank, per-layer NCCL gradient all-reduce overlapped with backward.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl  # noqa: E402

METRIC = "samples/sec under fixed memory budget, dynamic seq len, 1/2/4/8 B200"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="mimose", choices=["mimose", "reference"])
    ap.add_argument("--config", default="bert-base", choices=sorted(wl.CONFIGS))
    ap.add_argument("--no-baselines", action="store_true", help="skip static-plan / no-ckpt arms")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--simt", action="store_true", help="SIMT GEMMs instead of tcgen05")
    ap.add_argument("--gemm-mode", type=int, default=-1, help="tcgen05 GEMM variant (debug_options)")
    ap.add_argument("--granularity", type=int, default=0, choices=[0, 1],
                    help="checkpoint units of the headline arm: 0 layers (paper, A14), 1 attention/FFN blocks (A30)")
    ap.add_argument("--zero1", action="store_true",
                    help="ZeRO-1 optimizer-state sharding (SURVEY f4; needs world > 1 or --comm-force)")
    ap.add_argument("--comm-force", action="store_true",
                    help="build the NCCL communicator even at one GPU (a 1-rank communicator)")
    ap.add_argument("--planner", default="greedy", choices=["greedy", "exact", "knapsack"],
                    help="Algorithm 1 (default), the exact fewest-recompute planner (A29) or the "
                         "recompute-time-weighted exact planner (A31)")
    ap.add_argument("--p-drop", type=float, default=None,
                    help="override the dropout probability (experiments only: the headline keeps the config's)")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
            "sm_max_mhz": 1965.0}, "fallback"


def gemm_traffic():
    """DRAM bytes (read + write) per GEMM launch, from the committed ncu pass
    over this bench (tools/gemm_traffic.py -> profiles/<round>/gemm_traffic.json)."""
    import glob
    fs = sorted(glob.glob(os.path.join(ROOT, "profiles", "*", "gemm_traffic.json")))
    if not fs:
        return None, None
    d = json.load(open(fs[-1]))
    return d["dram_bytes_per_launch"], os.path.relpath(fs[-1], ROOT) + ": " + d["how"]


class Clocks:
    """nvidia-smi sampler for the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, dev: int):
        self.dev, self.rows, self.stop = dev, [], threading.Event()

    def _nvml_row(self, nv, h):
        r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
        bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
        return [str(self.dev), str(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)),
                str(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)),
                str(nv.nvmlDeviceGetPowerUsage(h) / 1000.0), hex(r)] + \
               ["Active" if r & b else "Not Active" for b in bits]

    def _run(self):
        # NVML in-process (a sample every ~20 ms, so a sub-second timed region
        # still gets many samples); nvidia-smi subprocess as the fallback
        nv = h = None
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.dev)
        except Exception:
            nv = None
        while not self.stop.is_set():
            try:
                if nv is not None:
                    self.rows.append(self._nvml_row(nv, h))
                else:
                    out = subprocess.run(["nvidia-smi", "-i", str(self.dev), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits"], capture_output=True,
                                         text=True, timeout=5).stdout.strip()
                    if out:
                        self.rows.append([t.strip() for t in out.split(",")])
            except Exception:
                pass
            self.stop.wait(0.02 if nv is not None else 0.2)
        self.source = "nvml" if nv is not None else "nvidia-smi"

    def __enter__(self):
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in self.rows for n, v in zip(names, r[5:9]) if v.lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows), "source": getattr(self, "source", None)}


def step_flops(cfg, n_seqs, S, St=0):
    """Algorithmic FLOPs of one step: model = 3 x forward
    (+ the LM head), and the forward FLOPs of one layer (added per dropped layer).
    Encoder-decoder: encoder layers at T_s, decoder layers (self + cross
    attention + FFN) at T_t, LM head at T_t; the per-layer figure is the mean."""
    H, F, T = cfg.hidden, cfg.ffn, n_seqs * S
    if cfg.arch == wl.ARCH_ENCDEC:
        Tt = n_seqs * St
        enc = 2.0 * T * (4 * H * H + 2 * H * F) + 4.0 * n_seqs * S * S * H
        dec = (2.0 * Tt * (4 * H * H + 2 * H * F) + 2.0 * n_seqs * St * St * H          # self (causal)
               + 2.0 * Tt * 2 * H * H + 2.0 * T * 2 * H * H + 4.0 * n_seqs * St * S * H)  # cross
        model = 3.0 * (enc * cfg.n_layers + dec * cfg.n_dec_layers + 2.0 * Tt * H * cfg.vocab)
        return model, (enc * cfg.n_layers + dec * cfg.n_dec_layers) / (cfg.n_layers + cfg.n_dec_layers)
    attn = 4.0 * n_seqs * S * S * H * (0.5 if cfg.arch == wl.ARCH_PRE_LN else 1.0)
    layer = 2.0 * T * (4 * H * H + 2 * H * F) + attn
    model = 3.0 * layer * cfg.n_layers
    if cfg.head == wl.HEAD_LM:
        model += 3.0 * 2.0 * T * H * cfg.vocab
    return model, layer


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# ---------------------------------------------------------------------------
# reference arm: the fp64 CPU oracle (DESIGN "Measurement")
# ---------------------------------------------------------------------------

def oracle_sample_step(cfg, S_longest, n_q, step, n_layers=None):
    """One oracle training step (forward, backward, AdamW) on a bounded sample:
    n_q questions of the workload through a model of n_layers encoder layers
    (default: all) whose word-embedding table shrinks in the same proportion,
    so every part of the step (layers, embedding, AdamW over the parameters)
    scales by n_layers / L.  Returns (seconds, samples processed)."""
    from oracle import model as om
    L = cfg.n_layers if n_layers is None else n_layers
    V = cfg.vocab if L == cfg.n_layers else max(1024, cfg.vocab * L // cfg.n_layers)
    sub = wl.small_config(cfg.name, n_seqs=n_q * (cfg.n_choices if cfg.head == wl.HEAD_MC else 1), n_layers=L,
                          vocab=V)
    params = ORACLE_PARAMS.setdefault((cfg.name, L), wl.init_params(sub))
    b = wl.make_batch(sub, S_longest, seed=wl.batch_seed(cfg, step))
    t0 = time.perf_counter()
    loss, G = om.train_step_grads(sub, params, b, wl.dropout_seed(cfg), step + 1)
    zeros = {k: np.zeros_like(v, np.float64) for k, v in G.items()}
    om.adamw(params, G, zeros, dict(zeros), 1, 1e-4)
    return time.perf_counter() - t0, n_q if cfg.head == wl.HEAD_MC else b.n_seqs


ORACLE_PARAMS: dict = {}


def cpu_baseline(cfg, n_steps=2, n_q=2):
    S = wl.roundup((cfg.seq_lo + cfg.seq_hi) // 2, cfg.pad)
    tot_t, tot_s = 0.0, 0
    for i in range(n_steps):
        t, s = oracle_sample_step(cfg, S, n_q, i)
        tot_t += t
        tot_s += s
    unit = "questions" if cfg.head == wl.HEAD_MC else "sequences"
    return {"value": tot_s / tot_t, "unit": "samples/s", "cores": len(os.sched_getaffinity(0)),
            "kind": "oracle",
            "sample": f"{n_steps} fp64 numpy training step(s) of {n_q} {unit} at S_pad={S} "
                      f"({cfg.name}, full width/depth), {tot_t:.1f} s"}


REF_BUDGET_S = 150.0   # the reference arm's whole --steps K --warmup W run


def run_reference(args):
    """--impl reference: the fp64 oracle as it stands, on the host cores, on a
    bounded sample per step.  A step is one question (MC) / sequence through the
    full model when K + W such steps fit REF_BUDGET_S; otherwise through a
    model with L_s of the L encoder layers and an L_s / L word-embedding table
    (every part of the step then scales by f = L_s / L: the L identical layers,
    the embedding and the AdamW sweep), L_s the largest that fits, counted as
    f of a sample."""
    world, rank, _ = dist_env()
    if rank != 0:
        return
    cfg = wl.CONFIGS[args.config]
    sched = wl.length_schedule(cfg, args.warmup + args.steps + 1)
    n_q = 1
    L = cfg.n_layers
    t_cal, _ = oracle_sample_step(cfg, sched[0], n_q, 0)           # calibration: one full-model step
    n = args.warmup + args.steps
    L_s = L if n * t_cal <= REF_BUDGET_S else max(1, int(L * REF_BUDGET_S / (n * t_cal)))
    for i in range(args.warmup):
        oracle_sample_step(cfg, sched[1 + i], n_q, 1 + i, L_s)
    tot_t, tot_s = 0.0, 0.0
    for i in range(args.steps):
        t, s_ = oracle_sample_step(cfg, sched[1 + args.warmup + i], n_q, 1 + args.warmup + i, L_s)
        tot_t += t
        tot_s += s_ * L_s / L
    v = tot_s / tot_t
    sample = (f"per step {n_q} question(s) of the {cfg.name} workload at the schedule's S_t through "
              f"{L_s} of {L} encoder layers with a {L_s}/{L} word-embedding table (+ head, AdamW), counted as "
              f"{L_s}/{L} of a sample; "
              f"fp64 numpy; calibration full-model step {t_cal:.2f} s")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "samples/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * tot_t / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": cfg.name},
            "cpu_baseline": {"value": v, "unit": "samples/s", "cores": len(os.sched_getaffinity(0)),
                             "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# Mimose arm
# ---------------------------------------------------------------------------

def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb

    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cfg = wl.CONFIGS[args.config]
    if args.p_drop is not None:
        cfg = dataclasses.replace(cfg, p_drop=args.p_drop)
    stream = torch.cuda.current_stream()
    use_tc = 0 if args.simt else 1
    if args.gemm_mode >= 0:
        mb.debug_options(gemm_mode=args.gemm_mode)

    # ---- budget (D2 / reading A21) from the library's own allocation sequence ----
    probe_ctx = mb.Mimose(cfg, 0, world=world, zero1=1 if args.zero1 else 0)
    C0 = probe_ctx.stats()["persistent_bytes"]
    ed = cfg.arch == wl.ARCH_ENCDEC
    dmax = cfg.max_seq if ed else None
    P0 = probe_ctx.dry_run(cfg.n_seqs, cfg.max_seq, [], dec_len=dmax)
    LB = probe_ctx.dry_run(cfg.n_seqs, cfg.max_seq, range(cfg.n_layers + cfg.n_dec_layers), dec_len=dmax)
    M = max(C0 + int(cfg.budget_frac * (P0 - C0)), LB)
    probe_ctx.close()

    def fresh_nccl_id():
        # one ncclUniqueId per communicator: every library context (one per arm)
        # bootstraps its own, so rank 0 draws a new id and broadcasts it each time
        if world == 1:
            return None
        t = torch.zeros(128, dtype=torch.uint8, device="cuda")
        if rank == 0:
            t.copy_(torch.frombuffer(bytearray(mb.nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(t, 0)
        return bytes(t.cpu().numpy().tolist())

    def new_ctx(budget, slab_bytes, enforce=1, **kw):
        kw.setdefault("zero1", 1 if args.zero1 else 0)
        kw.setdefault("comm_force", 1 if args.comm_force else 0)
        slab = torch.empty(slab_bytes, dtype=torch.uint8, device="cuda")
        ctx = mb.Mimose(cfg, budget, slab=slab, stream=stream, rank=rank, world=world,
                        nccl_id=fresh_nccl_id(), enforce_budget=enforce, use_tc=use_tc, **kw)
        ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
        # AdamW per gradient bucket on a side stream, overlapping the backward
        ctx.set_optimizer(1e-5, fused=True)
        if args.planner == "exact":
            ctx.set_planner(mb.PLANNER_EXACT)
        elif args.planner == "knapsack":
            ctx.set_planner(mb.PLANNER_EXACT_TIME)
        return ctx

    n_total = args.warmup + args.steps
    sched = wl.length_schedule(cfg, 10 + n_total)      # shared by every rank (same S_t)

    def host_batches(offset):
        return [wl.make_batch(cfg, sched[offset + i], seed=wl.batch_seed(cfg, offset + i, rank))
                for i in range(n_total)]

    def arrays(b):
        xs = [b.input_ids, b.token_type, b.lengths, b.labels]
        return xs + ([b.dec_ids, b.dec_lengths] if b.dec_ids is not None else [None, None])

    def to_dev(b):
        return [torch.tensor(np.ascontiguousarray(x, np.int32)).cuda() if x is not None else None for x in arrays(b)]

    def plan_for(ctx, b):
        return ctx.plan(*b.input_size2) if ed else ctx.plan(b.input_size)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def timed(ctx, batches, mode, plan_fixed=None, host=False, clocks=None, probe=False):
        """Runs warm-up then the timed steps; returns device ms (max over ranks)."""
        dev = None if host else [to_dev(b) for b in batches]
        pinned = None
        if host:
            pinned = []
            for b in batches:
                ts = [torch.from_numpy(np.ascontiguousarray(x, np.int32)).pin_memory() if x is not None else None
                      for x in arrays(b)]
                pinned.append(ts)

        def one(i):
            b = batches[i]
            t = pinned[i] if host else dev[i]
            bs = mb.Mimose.batch_struct(*t[:4], b.n_seqs, b.seq_len, host, t[4], t[5], b.dec_len)
            if mode == "mimose":
                p = plan_for(ctx, b)
            elif mode == "static":
                p = plan_fixed
            else:
                p = None
            ctx.forward(bs, p, want_loss=host)
            ctx.backward()
            ctx.step(1e-5)

        for i in range(args.warmup):
            one(i)
        barrier()
        if probe:
            ctx.probe(1)
        launches0 = ctx.stats()["kernel_launches"]
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        if clocks:
            clocks.__enter__()
        for i in range(args.warmup, n_total):
            one(i)
        ev1.record(stream)
        barrier()
        if clocks:
            clocks.__exit__()
        ms = ev0.elapsed_time(ev1)
        launches = ctx.stats()["kernel_launches"] - launches0
        pr = ctx.probe_read() if probe else None
        if probe:
            ctx.probe(0)
        if world > 1:
            t = torch.tensor([ms], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms, launches, pr

    samples_per_step = cfg.samples_per_step * world

    def sheltered(ctx, sched_, seed_base):
        """The sheltered phase: collect until the estimator is fitted;
        device time by CUDA events on the compute stream (host batches: the
        collector copies them in), samples processed."""
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        e0.record(stream)
        n = 0
        while ctx.phase == mb.PHASE_SHELTERED:
            b = wl.make_batch(cfg, sched_[n % len(sched_)], seed=wl.batch_seed(cfg, seed_base + n, rank))
            ctx.collect(ctx.host_batch(b), want_loss=False)
            ctx.backward()
            ctx.step(1e-5)
            n += 1
        e1.record(stream)
        barrier()
        return e0.elapsed_time(e1), n

    def tokens(batches):
        """(mean S_pad, padded tokens, valid tokens); encoder-decoder: source + target."""
        bs = batches[args.warmup:]
        return (float(np.mean([b.seq_len for b in bs])), int(sum(b.n_seqs * (b.seq_len + b.dec_len) for b in bs)),
                int(sum(int(b.lengths.sum()) + (int(b.dec_lengths.sum()) if b.dec_lengths is not None else 0)
                        for b in bs)))

    # ---- Mimose: sheltered phase, then the timed responsive steps ----
    ctx = new_ctx(M, M, granularity=args.granularity)
    t0 = time.perf_counter()
    sh_ms, sh_n = sheltered(ctx, sched, 10**6)
    sheltered_s = time.perf_counter() - t0
    batches = host_batches(10)
    clocks = Clocks(local)
    ms, launches, _ = timed(ctx, batches, "mimose", clocks=clocks)
    st = ctx.stats()
    # roofline pass: the same steps again with a CUDA-event pair around every GEMM launch
    ms_probe, _, pr = timed(ctx, batches, "mimose", probe=True)
    value = samples_per_step * args.steps / (ms / 1000.0)
    # e2e: host buffers through the public API; H2D + loss D2H inside the timed region
    ms_e2e, _, _ = timed(ctx, batches, "mimose", host=True)
    e2e = samples_per_step * args.steps / (ms_e2e / 1000.0)
    per_step_h2d = int(np.mean([sum(x.size for x in arrays(b) if x is not None) * 4 for b in batches]))
    st2 = ctx.stats()
    dropped, pred_err, flops_model, flops_hw = [], [], 0.0, 0.0
    for b in batches[args.warmup:]:
        p = plan_for(ctx, b)
        dropped.append(p.n_dropped)
        # prediction error as the paper defines it, on the whole-step peak:
        # the estimator's predicted peak for the plan vs the arena's exact peak
        actual = ctx.dry_run(b.n_seqs, b.seq_len, p.dropped, dec_len=b.dec_len if ed else None)
        pred_err.append(abs(p.predicted_peak - actual) / actual)
        fm, fr = step_flops(cfg, b.n_seqs, b.seq_len, b.dec_len)
        flops_model += fm
        flops_hw += fm + fr * p.n_dropped
    samples = [ctx.sample(j) for j in range(st["n_samples"])]
    t_ms = [np.mean(s["t_ms"]) for s in samples]
    mean_s, tok_pad, tok_valid = tokens(batches)

    pk, kind = peaks()
    gemm_ms, gemm_flops, gemm_n = pr
    tc = use_tc == 1 and mb.tc_gemm_available()
    ck = clocks.summary()
    at_max = bool(ck.get("sm_mhz") and ck.get("sm_max_mhz") and ck["sm_mhz"] >= 0.95 * ck["sm_max_mhz"])
    achieved = gemm_flops / (gemm_ms / 1000.0) / 1e12 if gemm_ms > 0 else 0.0
    if tc:
        # a run at max clock is judged against the burst peak, a clock-capped one
        # against the sustained (power-capped) peak (B200_PROFILING.md)
        burst, sust = float(pk["bf16_tflops"]), float(pk.get("bf16_tflops_sustained", pk["bf16_tflops"]))
        bound, unit = "tensor", "TFLOP/s"
        peak = burst if at_max else sust
        peak_note = (f"bf16_tflops ({kind}, burst: the timed region ran at {ck.get('sm_mhz')} MHz = max clock)"
                     if at_max else f"bf16_tflops_sustained ({kind}: clocks below max under load)")
        fracs = {"frac_vs_burst": achieved / burst, "frac_vs_sustained": achieved / sust}
    else:
        # SIMT fp32 FMA: 148 SMs x 128 lanes x 2 FLOP x sm_max clock
        peak = 148 * 128 * 2 * float(pk.get("sm_max_mhz", 1965.0)) * 1e6 / 1e12
        bound, unit = "alu", "TFLOP/s"
        peak_note = f"FP32 FMA: 148 SM x 128 lanes x 2 x {pk.get('sm_max_mhz', 1965.0)} MHz ({kind} clock)"
        fracs = {}
    traffic, traffic_src = gemm_traffic()
    roofline = {"bound": bound, "achieved": achieved, "peak": peak, "unit": unit,
                "frac": achieved / peak if peak else None, **fracs, "traffic": traffic, "traffic_source": traffic_src,
                "kernel": "GEMM (all linear layers: fwd, dgrad, wgrad)",
                "peak_source": peak_note, "launches": gemm_n,
                "share_of_step": gemm_ms / ms_probe if ms_probe else None,
                "measured": "CUDA events around each GEMM on the compute stream, separate pass over the same timed steps",
                "flops_per_launch": gemm_flops / max(gemm_n, 1)}
    ms_s_step = ms / args.steps
    sh_samples = samples_per_step * sh_n
    result = {
        "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_s_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16" if cfg.dtype == "bf16" else "f32",
        "data": "synthetic",
        "config": {"workload": cfg.name, "task": "translation-like encoder-decoder (UN_PC-like lengths)" if ed else
                   {wl.HEAD_MC: "SWAG-like multiple choice", wl.HEAD_QA: "span QA",
                    wl.HEAD_LM: "causal LM"}.get(cfg.head, "seq-cls"),
                   "batch_per_gpu": cfg.n_seqs, "samples_per_gpu_step": cfg.samples_per_step,
                   "seq_len": f"U[{cfg.seq_lo},{cfg.seq_hi}] pad {cfg.pad}", "budget_frac": cfg.budget_frac,
                   "budget_rule": "A21 (R2): M = max(C + f (P(empty, x_max) - C), LB(x_max))",
                   "budget_bytes": M, "persistent_bytes": C0, "no_ckpt_peak_at_max": P0,
                   "lower_bound_at_max": LB, "parallelism": f"dp{world}",
                   "l2": "no flush: per-step working set (weights+grads+optimizer >= 1.9 GB, activations) >> 126 MB L2",
                   "gemm": "tcgen05" if tc else "simt", "p_drop": cfg.p_drop,
                   **({"p_drop_override": True} if args.p_drop is not None else {})},
        "tokens": {"mean_seq_pad": mean_s, "padded_tokens_per_s": tok_pad * world / (ms / 1000.0),
                   "valid_tokens_per_s": tok_valid * world / (ms / 1000.0),
                   "valid_fraction": tok_valid / tok_pad},
        "incl_sheltered": {"value": (sh_samples + samples_per_step * args.steps) / ((sh_ms + ms) / 1000.0),
                           "sheltered_iters": sh_n, "sheltered_ms": sh_ms,
                           "note": "Tab. III charges the collector: the sheltered phase (host batches, "
                                   "shuttled forwards) + the timed steps, device time"},
        "roofline": roofline,
        "e2e": {"value": e2e, "unit": "samples/s", "h2d_bytes_per_step": per_step_h2d, "d2h_bytes_per_step": 4},
        "gpu_launches": launches,
        "clocks": ck,
        "mimose": {"planner": args.planner, "granularity": "sublayer" if args.granularity else "layer",
                   "violations": st2["violations"], "peak_bytes_max": st2["max_peak_bytes"],
                   "budget_bytes": M, "mean_layers_dropped": float(np.mean(dropped)),
                   "plan_cache_hits": st2["plan_cache_hits"], "plan_cache_misses": st2["plan_cache_misses"],
                   "planner_us_total": st2["planner_us_total"], "sheltered_iters": st2["collect_steps"],
                   "shuttled_iters": st2["shuttled_steps"], "sheltered_s": sheltered_s,
                   "collector_layer_fwd_ms_mean": float(np.mean(t_ms)) if t_ms else None,
                   "prediction_error_mean": float(np.mean(pred_err)), "prediction_error_max": float(np.max(pred_err))},
        "mfu": flops_model * world / (ms / 1000.0) / 1e12 / peak if tc else None,
        "hfu": flops_hw * world / (ms / 1000.0) / 1e12 / peak if tc else None,
        "tflops_model": flops_model * world / (ms / 1000.0) / 1e12,
    }
    ctx.close()
    del ctx
    torch.cuda.empty_cache()

    def arm(budget, batches_, sched_, granularity=0, planner=None, fixed=None, slab=None, enforce=1, **kw):
        """One same-run comparison arm: its own context (sheltered phase on
        sched_ unless a fixed plan / none), timed on batches_."""
        ctx = new_ctx(budget, slab or budget, enforce=enforce, granularity=granularity, **kw)
        if planner is not None:
            ctx.set_planner(planner)
        out = {}
        if fixed != "none":
            sms, sn = sheltered(ctx, sched_, 2 * 10**6)
            out["sheltered_ms"] = sms
        if fixed == "static":
            p = ctx.plan(cfg.n_seqs * cfg.max_seq, cfg.n_seqs * cfg.max_seq if ed else None)
            ms_a, _, _ = timed(ctx, batches_, "static", plan_fixed=p)
            out["layers_dropped"] = p.n_dropped
        elif fixed == "all":
            p = mb.Plan()
            p.drop_mask = (1 << ctx.n_units) - 1
            ms_a, _, _ = timed(ctx, batches_, "static", plan_fixed=p)
            out["layers_dropped"] = ctx.n_units
        elif fixed == "none":
            ms_a, _, _ = timed(ctx, batches_, "none")
        else:
            ms_a, _, _ = timed(ctx, batches_, "mimose")
            out["mean_dropped"] = float(np.mean([plan_for(ctx, b).n_dropped for b in batches_[args.warmup:]]))
        sta = ctx.stats()
        out.update(value=samples_per_step * args.steps / (ms_a / 1000.0), ms_per_step=ms_a / args.steps,
                   violations=sta["violations"], peak_bytes_max=sta["max_peak_bytes"])
        ctx.close()
        del ctx
        torch.cuda.empty_cache()
        return out, ms_a

    if not args.no_baselines:
        # static largest-input plan (Sublinear-style conservatism)
        result["static_plan"], ms_s = arm(M, batches, sched, fixed="static")
        # no checkpointing, budget not enforced (reports the peak it needs)
        result["no_ckpt"], ms_n = arm(M, batches, sched, fixed="none", slab=P0 + (1 << 20), enforce=0)
        result["no_ckpt"]["over_budget"] = result["no_ckpt"]["peak_bytes_max"] > M
        # all checkpointed: every layer dropped (the memory lower bound)
        result["all_ckpt"], ms_a = arm(M, batches, sched, fixed="all")
        result["all_ckpt"]["recompute_ratio"] = ms_a / ms_n
        # sub-layer checkpoint units (reading A30): attention / FFN
        # blocks planned independently by the same Algorithm 1, same budget
        if not ed:
            u, ms_u = arm(M, batches, sched, granularity=1)
            u.update(units=2 * cfg.n_layers, recompute_ratio=ms_u / ms_n)
            result["sublayer_units"] = u
        # the Knapsack (reading A31): units planned by least total
        # recompute time (the collector's t_l(x)), same budget (encoder-decoder: layers)
        k, ms_k = arm(M, batches, sched, granularity=0 if ed else 1, planner=mb.PLANNER_EXACT_TIME)
        k.update(units=cfg.n_layers + cfg.n_dec_layers if ed else 2 * cfg.n_layers, recompute_ratio=ms_k / ms_n)
        result["knapsack_units" if not ed else "knapsack_layers"] = k
        # the literal "f x no-checkpoint peak" budget, if feasible
        M_lit = int(cfg.budget_frac * P0)
        if M_lit >= LB:
            lit, ms_l = arm(M_lit, batches, sched)
            lit.update(budget_bytes=M_lit, recompute_ratio=ms_l / ms_n,
                       rule="M = f x P(empty, x_max) (literal north_star reading)")
            # the same tight budget with attention / FFN units planned by least
            # recompute time (A30 + A31): what the finer units buy when half the layers must go
            lk, ms_lk = arm(M_lit, batches, sched, granularity=0 if ed else 1, planner=mb.PLANNER_EXACT_TIME)
            lk.update(recompute_ratio=ms_lk / ms_n, units=cfg.n_layers + cfg.n_dec_layers if ed else 2 * cfg.n_layers)
            lit["knapsack_units" if not ed else "knapsack_layers"] = lk
            result["literal_budget"] = lit
        else:
            result["literal_budget"] = {"infeasible": True, "budget_bytes": M_lit, "lower_bound": LB}
        # the paper-like truncated-normal length schedule, own no-ckpt reference
        nsched = wl.length_schedule(cfg, 10 + n_total, kind="normal")
        nb = [wl.make_batch(cfg, nsched[10 + i], seed=wl.batch_seed(cfg, 5 * 10**6 + i, rank)) for i in range(n_total)]
        nm, ms_nm = arm(M, nb, nsched)
        nn, ms_nn = arm(M, nb, nsched, fixed="none", slab=P0 + (1 << 20), enforce=0)
        nm.update(schedule="truncated normal mu=(lo+hi)/2 sigma=(hi-lo)/4", mean_seq_pad=tokens(nb)[0],
                  no_ckpt_value=nn["value"], recompute_ratio=ms_nm / ms_nn)
        result["normal_schedule"] = nm
        # the multi-GPU code path on this one GPU: a 1-rank NCCL communicator with
        # ZeRO-1 (per-bucket reduce-scatter, sharded AdamW, weight all-gather)
        if world == 1 and not ed:
            z, ms_z = arm(M, batches, sched, comm_force=1, zero1=1)
            z.update(note="comm_force=1, zero1=1 at world 1: the DP/ZeRO-1 collectives run on a 1-rank "
                          "communicator", overhead_vs_headline=ms_z / ms)
            result["zero1_nccl_1rank"] = z
        result["recompute_ratio"] = ms / ms_n
        result["speedup_vs_static"] = ms_s / ms
        result["paper_context"] = ("V100 (P:227): Mimose ~18.0% faster than Sublinear, ~15.0% than DTR "
                                   "(P:252-254); 2.6% slower than no-checkpoint at 8 GB (P:258)")

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            result["cpu_baseline"] = cpu_baseline(cfg)
        except Exception as e:  # never let the reported baseline kill the line
            result["cpu_baseline"] = {"value": None, "error": str(e)[:200], "kind": "oracle"}
    if rank == 0:
        print(json.dumps(result), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
