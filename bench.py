#!/usr/bin/env python
"""Benchmark of the INSTA hot path on B200 (driver contract: one JSON line on rank 0).

A step = one full evaluation of the hot path on the 15M-pin synthetic graph
(BASELINE.json configs[3], "C4"): insta_forward (arrival propagation over all
levels + endpoint slack + WNS/TNS) followed by insta_backward (dTNS/d(arc
mean) for every arc).  value = pins processed per second (whole job: N ranks x
pins / max-over-ranks step time).  With N > 1 each rank evaluates its own
independent replica of the same graph (weak scaling; no data-path collective,
one all_reduce of the timing at the end); the C5 batched leg shards 1024
scenarios over the ranks.  `--gpus N` without torchrun re-launches itself
with torch.distributed.run (one process per GPU).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--tau 0] [--schedule 0]
  python bench.py --impl reference ...   # the fp64 CPU oracle on the box's host cores
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

from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

METRIC = "fwd+bwd pins/s on 15M-pin graph (insta_forward + insta_backward, TNS gradient)"
UNIT = "pins/s"


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 8:
                self.rows.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        rows = self.rows
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}

        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [num(r[0]) for r in rows if num(r[0]) is not None]
        mx = [num(r[1]) for r in rows if num(r[1]) is not None]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[4 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


# ---------------------------------------------------------------------------
# byte model: algorithmic bytes per launch
# ---------------------------------------------------------------------------
HEAVY_FANOUT = 256   # csrc/internal.h kHeavyFanout: drivers above it use the atomic path


def survey_bytes(N, E, P, lse):
    """SURVEY.md §8(d) algorithmic bytes (fp32 16 B state, 20 B arc record; the roofline's model):
    forward 20 B/pin + 36 B/arc (+8 B/arc Eq 6 weights in LSE) + 32 B/endpoint;
    backward (mean channel, stored weights) 12 B/pin + 28 B/arc + 12 B/endpoint."""
    fwd = 20 * N + (44 if lse else 36) * E + 32 * P
    bwd = 12 * N + 28 * E + 12 * P
    return fwd, bwd


def sched0_bytes(sc, N, E, n_src, P, nnz_arcs, lse):
    """Bytes the default schedule's kernels move (this layout): forward (entry-parallel
    sweep fwdx_kernel, folded pins kept in registers) 8 B/head (row, pin) + per entry 20 B (source
    word, record of e) + a 32 B source-record gather + 20 B/folded pin (word, record of e') + a 32 B
    record store per head + arg-max 4 B/head (hard) or Eq 6 weights 16 B/entry (LSE) + 16 B/startpoint
    + 41 B/endpoint (slack); backward (sweep) 8 B/arc zero fill + 25 B/endpoint seeds + per head
    52 B (row 4, seed 8, arg-max 4, accumulator read + clear 32; LSE: no arg-max) + per entry 20 B
    topology (+16 B weights in LSE) + 16 B share pushed + 8 B per nonzero gradient."""
    H, X, F = sc["num_heads"], sc["num_entries"], sc["num_folded"]
    fwd = (8 * H + 20 * X + 32 * X + 20 * F + 32 * H + (16 * X if lse else 4 * H) + 16 * n_src + 41 * P)
    bwd = (8 * E + 25 * P + (48 if lse else 52) * H + (36 if lse else 20) * X + 16 * X + 8 * nnz_arcs)
    return fwd, bwd


def topk_bytes(g, K):
    """insta_topk_forward: per non-source pin a row pointer; per arc its source word and
    record (20 B); per (arc, sink rf, source transition) the parent's K queue slots ({mu, var} 16 B +
    startpoint 4 B); every (pin, rf) writes its K slots."""
    N, E = int(g.num_pins), int(g.num_arcs)
    n_src = int(np.count_nonzero(np.bincount(g.arc_to, minlength=N) == 0))
    n_non = int(np.count_nonzero(g.arc_unate == 2))
    return 4 * (N - n_src) + 20 * E + (2 * E + 2 * n_non) * K * 20 + 2 * N * K * 20


def cpu_oracle_sample(cfg_name, sample_pins, tau, omp=False, g=None):
    """fp64 CPU oracle fwd + slack + bwd on the workload (or a bounded sample of it: the same generator
    recipe -- depth, fanout law, endpoint fraction -- at `sample_pins` pins).  omp: the OpenMP
    level-parallel build of the same oracle on every host core."""
    import oracle  # test infrastructure: allowed in the cpu_baseline / reference leg only
    if g is None:
        g = synth.generate(cfg_name, pins=sample_pins)
    og = oracle.OGraph(g)
    t0 = time.perf_counter()
    f = oracle.forward(og, 3.0, tau, omp=omp)
    oracle.slack(og, f["A"])
    oracle.backward(og, 3.0, tau, omp=omp)
    dt = time.perf_counter() - t0
    return g.num_pins, dt


def host_info():
    cores = len(os.sched_getaffinity(0))
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return cores, model


def run_reference(args, rank, world):
    if rank != 0:
        return
    cfg = synth.CONFIGS[args.config]
    sample = args.ref_sample_pins
    times = []
    npins = 0
    for i in range(args.warmup + args.steps):
        npins, dt = cpu_oracle_sample(args.config, sample, args.tau)
        if i >= args.warmup:
            times.append(dt)
    T = float(np.sum(times))
    val = npins * len(times) / T
    cores, model = host_info()
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * T / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name} recipe, oracle sample of {npins} pins (full workload {cfg.pins} pins)",
                   "tau": args.tau, "n_sigma": 3.0},
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "cpu_model": model,
                         "host_cores": cores,
                         "sample": f"{npins}-pin graph from the {cfg.name} generator recipe, fwd+slack+bwd, 1 thread"},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def timed_passes(G, stream, dev, steps, tau, schedule, d_mean, flush=None):
    """CUDA-event time of insta_forward and insta_backward over `steps` passes on `stream`;
    flush: a callable run before each pass outside the timed events (cold L2)."""
    import torch
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(steps)]
    for k in range(steps):
        if flush is not None:
            flush()
        ev[k][0].record(stream)
        G.forward(3.0, tau, schedule, sync=False, stream=stream)
        ev[k][1].record(stream)
        G.backward(out=d_mean, stream=stream)
        ev[k][2].record(stream)
    torch.cuda.synchronize(dev)
    f = [ev[k][0].elapsed_time(ev[k][1]) for k in range(steps)]
    b = [ev[k][1].elapsed_time(ev[k][2]) for k in range(steps)]
    return float(np.mean(f)), float(np.mean(b)), float(np.median(f)), float(np.median(b))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="insta", choices=["insta", "reference"])
    ap.add_argument("--config", default="C4")
    ap.add_argument("--tau", type=float, default=0.0)
    ap.add_argument("--schedule", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--ref-sample-pins", type=int, default=1_500_000)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-full", type=int, default=1, help="cpu_baseline on the full workload (else the sample)")
    ap.add_argument("--batch-scenarios", type=int, default=1024, help="C5 batched evaluations (0 = skip)")
    ap.add_argument("--topk", type=int, default=32, help="Top-K CPPR propagation K (0 = skip)")
    ap.add_argument("--topk-wide", type=int, default=128, help="second Top-K leg, K > 32 (0 = skip)")
    ap.add_argument("--clark", type=int, default=1, help="time the Clark merge path (0 = skip)")
    ap.add_argument("--place", type=int, default=1, help="time Eq 7 / Eq 8 (0 = skip)")
    ap.add_argument("--lse", type=int, default=1, help="time the LSE (tau = 1 ps) fwd+bwd leg (0 = skip)")
    ap.add_argument("--cold", type=int, default=1, help="time fwd+bwd with L2 flushed before every pass (0 = skip)")
    ap.add_argument("--incremental", type=int, default=1,
                    help="time incremental re-annotation (a7): C4 small updates, C3 1%% steps (0 = skip)")
    ap.add_argument("--c3-steps", type=int, default=100)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # one process per GPU: re-launch under torch.distributed.run (rank 0 prints the line)
        import socket
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
        sys.exit(subprocess.call(cmd))

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import paper_conf_dac_lugklr25_b200 as insta

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)

    cfg = synth.CONFIGS[args.config]
    g = synth.generate(cfg)
    N, E, P = g.num_pins, g.num_arcs, g.num_endpoints
    G = insta.Graph(g, device=local)
    n_src = int(np.count_nonzero(np.bincount(g.arc_to, minlength=N) == 0))
    stream = torch.cuda.Stream(dev)
    d_mean = torch.empty((E, 2), dtype=torch.float32, device=dev)
    sched = G.schedule()
    peak, peak_kind = _peaks()

    # ---------------- the headline: C4 hard mode fwd+bwd, K timed passes -------------
    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            G.forward(3.0, args.tau, args.schedule, sync=False, stream=stream)
            G.backward(out=d_mean, stream=stream)
        stream.synchronize()
        s = G.summary(stream=stream)
        K = args.steps
        ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(K)]
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        clocks = ClockSampler(local)
        clocks.start()
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize(dev)
        e0.record(stream)
        for k in range(K):
            ev[k][0].record(stream)
            G.forward(3.0, args.tau, args.schedule, sync=False, stream=stream)
            ev[k][1].record(stream)
            G.backward(out=d_mean, stream=stream)
            ev[k][2].record(stream)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        if world > 1:
            torch.distributed.barrier()
        clk = clocks.stop()
        total_ms = e0.elapsed_time(e1)
        fwd_ms = float(np.mean([ev[k][0].elapsed_time(ev[k][1]) for k in range(K)]))
        bwd_ms = float(np.mean([ev[k][1].elapsed_time(ev[k][2]) for k in range(K)]))

    if world > 1:
        t = torch.tensor([total_ms, fwd_ms, bwd_ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        total_ms, fwd_ms, bwd_ms = (float(x) for x in t.tolist())
    ms_step = total_ms / args.steps
    value = world * N / (ms_step * 1e-3)

    # roofline: SURVEY §8(d) algorithmic bytes over the event-timed call; the dominant kernel
    lse = args.tau > 0
    dm = d_mean.cpu().numpy()
    nnz_arcs = int(np.count_nonzero((dm != 0).any(axis=1)))
    sfb, sbb = survey_bytes(N, E, P, lse)
    kfb, kbb = sched0_bytes(sched, N, E, n_src, P, nnz_arcs, lse)
    fwd_gbs, bwd_gbs = sfb / (fwd_ms * 1e-3) / 1e9, sbb / (bwd_ms * 1e-3) / 1e9
    dom = "fwd" if fwd_ms >= bwd_ms else "bwd"
    ach = fwd_gbs if dom == "fwd" else bwd_gbs
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(f"{args.config}_{dom}_tau{args.tau:g}_s{args.schedule}")
        except Exception:
            traffic = None
    roofline = {
        "bound": "hbm", "kernel": ("fwdx_kernel<entry-parallel sweep, parity dataflow> + slack_kernel (insta_forward)" if dom == "fwd"
                                   else "bwd_prep_kernel + bwdl_kernel<sweep> (insta_backward)"),
        "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak, "peak_kind": peak_kind,
        "traffic": traffic, "traffic_source": "profiles/traffic.json: ncu --set full dram__bytes_read.sum + "
                                              "dram__bytes_write.sum per launch, round 2",
        "byte_model": "SURVEY.md 8(d): fwd 20 B/pin + 36 B/arc + 32 B/endpoint (+8 B/arc LSE), "
                      "bwd 12 B/pin + 28 B/arc + 12 B/endpoint",
        "fwd_alg_bytes": sfb, "bwd_alg_bytes": sbb, "fwd_gbs": fwd_gbs, "bwd_gbs": bwd_gbs,
        "fwd_bwd_gbs": (sfb + sbb) / ((fwd_ms + bwd_ms) * 1e-3) / 1e9,
        "fwd_bwd_frac": (sfb + sbb) / ((fwd_ms + bwd_ms) * 1e-3) / 1e9 / peak,
        "kernel_layout_bytes": {"fwd": kfb, "bwd": kbb, "fwd_gbs": kfb / (fwd_ms * 1e-3) / 1e9,
                                "bwd_gbs": kbb / (bwd_ms * 1e-3) / 1e9,
                                "what": "bytes the default schedule's kernels move (bench.sched0_bytes, DESIGN.md §6)"},
    }

    # ---------------- LSE (tau = 1 ps): the differentiable mode (Eq 4, Eq 6) -------------
    lse_leg = None
    if args.lse and world == 1:
        with torch.cuda.stream(stream):
            for _ in range(3):
                G.forward(3.0, 1.0, args.schedule, sync=False, stream=stream)
                G.backward(out=d_mean, stream=stream)
            lf, lb, _, _ = timed_passes(G, stream, dev, max(5, min(args.steps, 10)), 1.0, args.schedule, d_mean)
            ls = G.summary(stream=stream)
        lfb, lbb = survey_bytes(N, E, P, True)
        lse_leg = {"tau": 1.0, "fwd_ms": lf, "bwd_ms": lb, "fwd_bwd_ms": lf + lb, "pins_per_s": N / ((lf + lb) * 1e-3),
                   "fwd_gbs": lfb / (lf * 1e-3) / 1e9, "bwd_gbs": lbb / (lb * 1e-3) / 1e9,
                   "fwd_frac": lfb / (lf * 1e-3) / 1e9 / peak, "bwd_frac": lbb / (lb * 1e-3) / 1e9 / peak,
                   "fwd_bwd_frac": (lfb + lbb) / ((lf + lb) * 1e-3) / 1e9 / peak, "tns": ls.tns, "wns": ls.wns}

    # ---------------- cold L2: a 512 MB write before every pass -------------
    cold = None
    if args.cold and world == 1:
        junk = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device=dev)

        def flush():
            junk.zero_()   # on the current stream (the pass's stream, below)

        with torch.cuda.stream(stream):
            cf, cb, cfm, cbm = timed_passes(G, stream, dev, max(5, min(args.steps, 10)), args.tau, args.schedule,
                                            d_mean, flush)
        del junk
        cold = {"what": "512 MB buffer written before every pass (L2 = 126 MB), events around the pass only",
                "fwd_ms": cf, "bwd_ms": cb, "fwd_bwd_ms": cf + cb,
                "fwd_bwd_frac": (sfb + sbb) / ((cf + cb) * 1e-3) / 1e9 / peak}

    # ---------------- end to end through the public API with host buffers -------------
    # Every step: H2D of all arc delays (mean, sigma; pinned host memory), insta_update_arcs (every arc),
    # insta_forward, insta_backward, insta_slack, and D2H of the full gradient + the endpoint slacks.
    # Steps are pipelined on three streams with double-buffered device staging: the H2D of step k+1 and
    # the D2H of step k-1 overlap step k's kernels (different copy directions, separate engines).
    e2e = None
    if args.e2e_steps > 0:
        m_h = torch.from_numpy(np.ascontiguousarray(g.arc_mean, np.float32)).pin_memory()
        s_h = torch.from_numpy(np.ascontiguousarray(g.arc_sigma, np.float32)).pin_memory()
        out_h = [torch.empty((E, 2), dtype=torch.float32).pin_memory() for _ in range(2)]
        sl_h = [torch.empty(P, dtype=torch.float32).pin_memory() for _ in range(2)]
        m_d = [torch.empty_like(m_h, device=dev) for _ in range(2)]
        s_d = [torch.empty_like(s_h, device=dev) for _ in range(2)]
        dm_d = [torch.empty((E, 2), dtype=torch.float32, device=dev) for _ in range(2)]
        sl_d = [torch.empty(P, dtype=torch.float32, device=dev) for _ in range(2)]
        s_in, s_out = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        ev_in = [torch.cuda.Event() for _ in range(2)]
        ev_in_free = [torch.cuda.Event() for _ in range(2)]
        ev_done = [torch.cuda.Event() for _ in range(2)]
        ev_out_free = [torch.cuda.Event() for _ in range(2)]
        for b in range(2):
            ev_in_free[b].record(stream)
            ev_out_free[b].record(stream)

        def e2e_step(k):
            b = k & 1
            with torch.cuda.stream(s_in):                  # H2D of this step's inputs
                s_in.wait_event(ev_in_free[b])
                m_d[b].copy_(m_h, non_blocking=True)
                s_d[b].copy_(s_h, non_blocking=True)
                ev_in[b].record(s_in)
            with torch.cuda.stream(stream):                # the public API calls
                stream.wait_event(ev_in[b])
                G.update_arcs(None, m_d[b], s_d[b], incremental=False, stream=stream)
                ev_in_free[b].record(stream)
                stream.wait_event(ev_out_free[b])
                G.forward(3.0, args.tau, args.schedule, sync=False, stream=stream)
                G.backward(out=dm_d[b], stream=stream)
                G.lib.insta_slack(G._h, sl_d[b].data_ptr(), None, stream.cuda_stream, None)
                ev_done[b].record(stream)
            with torch.cuda.stream(s_out):                 # D2H of this step's results
                s_out.wait_event(ev_done[b])
                out_h[b].copy_(dm_d[b], non_blocking=True)
                sl_h[b].copy_(sl_d[b], non_blocking=True)
                ev_out_free[b].record(s_out)

        for k in range(2):                                 # warm-up of the pipeline
            e2e_step(k)
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        for k in range(args.e2e_steps):
            e2e_step(k)
        torch.cuda.synchronize(dev)
        dt = (time.perf_counter() - t0) / args.e2e_steps
        tns_host = float(np.minimum(sl_h[(args.e2e_steps - 1) & 1].numpy().astype(np.float64), 0).sum())
        if world > 1:
            t = torch.tensor([dt], dtype=torch.float64, device=dev)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            dt = float(t.item())
        e2e = {"value": world * N / dt, "unit": UNIT, "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": int(E * 16), "d2h_bytes_per_step": int(E * 8 + P * 4),
               "tns_from_host_slack": tns_host,
               "what": "per step: H2D of every arc's mean/sigma from pinned memory, insta_update_arcs (all arcs), "
                       "insta_forward, insta_backward, insta_slack, D2H of the full gradient and the endpoint "
                       "slacks; steps pipelined over 3 streams (H2D k+1 and D2H k-1 overlap step k), "
                       f"{args.e2e_steps} steps, host wall clock"}

    # ---------------- end to end, incremental (the sizing loop's step): 1 % re-annotation -------------
    # Per step: H2D of the step's updated arcs (ids, mean, sigma from pinned memory), insta_update_arcs
    # (incremental), insta_forward with the summary read back (synchronous: the host decides the next
    # step on TNS), insta_backward into device memory (consumed on the device by insta_stage_gradients),
    # D2H of the endpoint slacks.  Host wall clock.  Runs on a copy of the annotation: restored after.
    e2e_inc = None
    if args.e2e_steps > 0 and world == 1:
        upd = [synth.sizing_step(g, 9000 + k, frac=0.01) for k in range(args.e2e_steps + 2)]
        pinned = [tuple(torch.from_numpy(np.ascontiguousarray(x)).pin_memory() for x in u) for u in upd]
        sl_h = torch.empty(P, dtype=torch.float32).pin_memory()
        sl_d = torch.empty(P, dtype=torch.float32, device=dev)
        h2d = 0
        with torch.cuda.stream(stream):
            G.forward(3.0, args.tau, args.schedule, stream=stream)
            for k, (ih, mh, sh) in enumerate(pinned):
                if k == 2:
                    torch.cuda.synchronize(dev)
                    t0 = time.perf_counter()
                ids = ih.to(dev, non_blocking=True)
                m = mh.to(dev, non_blocking=True)
                sg = sh.to(dev, non_blocking=True)
                if k >= 2:
                    h2d += ih.numel() * 4 + mh.numel() * 4 + sh.numel() * 4
                G.update_arcs(ids, m, sg, incremental=True, stream=stream)
                summ_k = G.forward(3.0, args.tau, args.schedule, stream=stream)
                G.backward(out=d_mean, stream=stream)
                G.lib.insta_slack(G._h, sl_d.data_ptr(), None, stream.cuda_stream, None)
                sl_h.copy_(sl_d, non_blocking=True)
            stream.synchronize()
            dt = (time.perf_counter() - t0) / args.e2e_steps
            # restore the original annotation for the legs that follow
            G.update_arcs(None, torch.as_tensor(g.arc_mean, device=dev), torch.as_tensor(g.arc_sigma, device=dev),
                          incremental=False, stream=stream)
            G.forward(3.0, args.tau, args.schedule, stream=stream)
        e2e_inc = {"value": N / dt, "unit": UNIT, "ms_per_step": dt * 1e3,
                   "h2d_bytes_per_step": int(h2d / args.e2e_steps), "d2h_bytes_per_step": int(P * 4 + 24),
                   "tns_last": summ_k.tns,
                   "what": "per step: H2D of a 1 % sizing update (synth.sizing_step: ids, mean, sigma), "
                           "insta_update_arcs(incremental), insta_forward + summary read (sync), insta_backward "
                           "(gradient stays on the device), D2H of the endpoint slacks; host wall clock"}

    # ---------------- batched scenarios (C5): 1024 evaluations sharded over the ranks -------------
    batched = None
    if args.batch_scenarios > 0:
        from paper_conf_dac_lugklr25_b200 import dist as idist
        nsc = args.batch_scenarios
        n_ocv = nsc // 2
        scs = synth.c5_scenarios(g, n=nsc, n_ocv=n_ocv)

        def is_sizing(sc):
            return sc.get("delta_arc") is not None and sc["n_sigma"] == 3.0 and sc["derate_cell"] == 1.0 \
                and sc["derate_net"] == 1.0

        packed = {}

        def ev(sub, want_grad):
            # OCV scenarios (and anything with derates): the batched kernels, 32 per pass; sizing candidates
            # (one cell's arcs re-annotated): the cone pass per candidate (insta_eval_candidates), their
            # arrays packed and uploaded once (not per timed call)
            with torch.cuda.stream(stream):
                if not want_grad and all(is_sizing(sc) for sc in sub):
                    key = (id(sub[0]), len(sub))
                    if key not in packed:
                        packed[key] = G.pack_candidates(sub, stream=stream)
                    return G.eval_packed(packed[key], stream=stream), None
                summ, dsum = G.forward_batch(sub, tau=args.tau, want_grad=want_grad, stream=stream)
            return summ, dsum

        dd = torch.distributed if world > 1 else None
        with torch.cuda.stream(stream):
            G.forward(3.0, args.tau, 0, stream=stream)   # the base state the candidates are evaluated against
            # warm-up: one untimed pass of the same calls (allocates the batch and staging buffers)
            idist.evaluate_sharded(ev, scs, n_ocv, E, rank, world, dev, dd)
            stream.synchronize()
            if world > 1:
                torch.distributed.barrier()
            b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            b0.record(stream)
            ctiming = {}
            summ_all, grad_sum = idist.evaluate_sharded(ev, scs, n_ocv, E, rank, world, dev, dd, timing=ctiming)
            b1.record(stream)
            torch.cuda.synchronize(dev)
            bms = b0.elapsed_time(b1)
        coll_ms = None
        if world > 1:
            t = torch.tensor([bms, ctiming.get("collective_ms", 0.0)], dtype=torch.float64, device=dev)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            bms, coll_ms = (float(x) for x in t.tolist())
        sa = summ_all.cpu().numpy()
        split = None
        if world == 1:   # the two halves timed separately (and the sizing half on the batched kernels too)
            with torch.cuda.stream(stream):
                t0, t1, t2, t3 = (torch.cuda.Event(enable_timing=True) for _ in range(4))
                t0.record(stream)
                ev(scs[:n_ocv], True)
                t1.record(stream)
                ev(scs[n_ocv:], False)
                t2.record(stream)
                G.forward_batch(scs[n_ocv:], tau=args.tau, want_grad=False, stream=stream)
                t3.record(stream)
                torch.cuda.synchronize(dev)
            split = {"ocv_fwd_bwd_ms": t0.elapsed_time(t1), "sizing_cone_ms": t1.elapsed_time(t2),
                     "sizing_batched_kernels_ms": t2.elapsed_time(t3),
                     "sizing_evals_per_s_cone": (nsc - n_ocv) / (t1.elapsed_time(t2) * 1e-3)}
        batched = {"workload": f"C5: {nsc} scenarios on the {cfg.name} graph ({n_ocv} OCV fwd+bwd with TNS-gradient "
                               f"sum, 32 scenarios per batched pass; {nsc - n_ocv} one-cell sizing candidates through "
                               f"the cone pass, insta_eval_candidates)", "split": split,
                   "evals": nsc, "ms": bms, "evals_per_s": nsc / (bms * 1e-3),
                   "pins_per_s": nsc * N / (bms * 1e-3), "n_gpus": world,
                   "collectives": "all_gather(per-scenario summaries) + all_reduce(SUM, gradient sum)" if world > 1
                   else "none (1 rank)", "collective_ms": coll_ms,
                   "tns_min": float(sa[:, 1].min()), "tns_max": float(sa[:, 1].max())}

    # ---------------- Top-K unique-startpoint propagation + CPPR slack -------------
    topk = None
    def topk_leg(K, warm, nk):
        torch.cuda.synchronize(dev)
        free0 = torch.cuda.mem_get_info(dev)[0]
        with torch.cuda.stream(stream):
            for _ in range(warm):
                G.topk_forward(K, 3.0, stream=stream)
                G.topk_slack(stream=stream, sync=False)
            stream.synchronize()
            t0, t1, t2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t0.record(stream)
            for _ in range(nk):
                G.topk_forward(K, 3.0, stream=stream)
            t1.record(stream)
            for _ in range(nk):
                G.topk_slack(stream=stream, sync=False)
            t2.record(stream)
            stream.synchronize()
            ts, _, _ = G.topk_slack(stream=stream)
        tf, tsl = t0.elapsed_time(t1) / nk, t1.elapsed_time(t2) / nk
        tk_mem = (free0 - torch.cuda.mem_get_info(dev)[0]) / 1e9   # queues + slack + lists (library cudaMalloc)
        tk_bytes = topk_bytes(g, K)
        return {"workload": f"{cfg.name}, Top-K = {K} unique-startpoint queues (Alg 1 + Alg 2) + CPPR slack against "
                            f"a per-(endpoint, startpoint) RAT table", "K": K, "fwd_ms": tf, "slack_ms": tsl,
                "pins_per_s": N / ((tf + tsl) * 1e-3), "alg_bytes": tk_bytes, "gbs": tk_bytes / (tf * 1e-3) / 1e9,
                "tns": ts.tns, "wns": ts.wns, "violations": ts.num_violations,
                "device_memory_gb_added": tk_mem}

    topk = topk_wide = None
    if args.topk > 0 and world == 1:
        G.set_cppr_rat(*synth.cppr_rat_table(g))
        topk = topk_leg(args.topk, 2, max(1, min(args.steps, 5)))
        topk["paper_context"] = ("PAPER.md Table I (L184-193): block-1 (15M pins) at TopK=32 in 0.39 s and 21.13 GB "
                                 "on 1x A100 (incl. its own slack); other hardware, other design")
        if args.topk_wide > 0:   # the paper's CPPR study configuration: K = 128
            topk_wide = topk_leg(args.topk_wide, 1, 2)
            topk_wide["device_memory_gb_state"] = 40.0 * args.topk_wide * N / 1e9
            topk_wide["what"] = ("wide-queue kernel (a warp per (pin, rf), queue in shared memory); memory added "
                                 "relative to the K = %d state it replaces" % args.topk)

    # ---------------- Clark moment-matching merge -------------
    clark = None
    if args.clark and world == 1:
        with torch.cuda.stream(stream):
            for _ in range(2):
                G.clark_forward(3.0, sync=False, stream=stream)
                G.clark_backward(stream=stream)
            stream.synchronize()
            nk = max(1, min(args.steps, 5))
            c0, c1, c2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            dcl = torch.empty((E, 2), dtype=torch.float32, device=dev)
            c0.record(stream)
            for _ in range(nk):
                G.clark_forward(3.0, sync=False, stream=stream)
            c1.record(stream)
            for _ in range(nk):
                G.lib.insta_clark_backward(G._h, None, dcl.data_ptr(), None, None, stream.cuda_stream)
            c2.record(stream)
            stream.synchronize()
            cs = G.clark_forward(3.0, stream=stream)
        cf, cb = c0.elapsed_time(c1) / nk, c1.elapsed_time(c2) / nk
        clark = {"workload": f"{cfg.name}, Clark moment-matching max (fp64, per-level launches) + slack, and its "
                             f"TNS backward", "fwd_ms": cf, "bwd_ms": cb, "pins_per_s": N / ((cf + cb) * 1e-3),
                 "tns": cs.tns, "wns": cs.wns, "violations": cs.num_violations}

    place = None
    if args.place and world == 1:   # NEXT 4: Eq 7 loss + gradient (insta_timing_loss), Eq 8 (insta_grad_norm_ratio)
        with torch.cuda.stream(stream):
            gen = torch.Generator(device=dev).manual_seed(77)
            px = torch.rand(N, generator=gen, device=dev) * 1000.0
            py = torch.rand(N, generator=gen, device=dev) * 1000.0
            aw = d_mean.abs().sum(dim=1).contiguous()          # per-arc TNS sensitivity (R21)
            gw = torch.rand(N, generator=gen, device=dev)
            for _ in range(2):
                L_, gx_, gy_ = G.timing_loss(px, py, aw, 1e-3, stream=stream)
                insta.grad_norm_ratio(gx_, gw, stream=stream)
            stream.synchronize()
            nk = max(1, min(args.steps, 10))
            p0, p1, p2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            p0.record(stream)
            for _ in range(nk):
                L_, gx_, gy_ = G.timing_loss(px, py, aw, 1e-3, stream=stream)
            p1.record(stream)
            for _ in range(nk):
                insta.grad_norm_ratio(gx_, gw, stream=stream)
            p2.record(stream)
            stream.synchronize()
        tl_ms, nr_ms = p0.elapsed_time(p1) / nk, p1.elapsed_time(p2) / nk
        # algorithmic bytes: Eq 7 reads x, y (8 B/pin) and writes the gradient (8 B/pin); per arc its two
        # ends and weight (12 B) and the two ends' positions (16 B); Eq 8 reads both vectors once
        tl_bytes = 16 * N + 28 * E
        place = {"workload": f"{cfg.name}: Eq 7 timing loss + gradient over every arc (weights |dTNS/dmean|, "
                             f"random positions), Eq 8 norm ratio over N pins",
                 "eq7_ms": tl_ms, "eq7_alg_gbs": tl_bytes / (tl_ms * 1e-3) / 1e9, "eq8_ms": nr_ms,
                 "eq8_gbs": 8 * N / (nr_ms * 1e-3) / 1e9, "loss": float(L_.item())}

    # ---------------- incremental re-annotation -------------
    # Runs last: it changes the graph's arcs.  Each step: insta_update_arcs (device buffers, incremental)
    # + insta_forward, CUDA events around both.  C4: small sizing updates (1 cell, ~1e-5, ~1e-4 of the arcs)
    # take the cone pass (default policy, include/insta.h cone_max), against update + full pass.  C3
    # (BASELINE configs[2]): 100 steps of 1 % sizing updates, default policy (a full pass: the cone of a
    # random 1 % update reaches every level) and the cone pass forced, against update + full pass.
    def inc_series(GG, gg, fracs_steps, modes, seed0):
        out = {}
        with torch.cuda.stream(stream):
            GG.forward(3.0, 0.0, 0, stream=stream)
            for frac, nst in fracs_steps:
                upd = [tuple(torch.as_tensor(x, device=dev) for x in synth.sizing_step(gg, seed0 + k, frac=frac))
                       for k in range(nst)]
                row = {"frac": frac, "arcs_per_step": int(np.mean([len(u[0]) for u in upd])), "steps": nst}
                for mode, cmax in modes:
                    ts, cone = [], []
                    for ids, m, sg in upd:
                        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        a0.record(stream)
                        GG.update_arcs(ids, m, sg, incremental=(mode != "full"), stream=stream)
                        GG.forward(3.0, 0.0, 0, sync=False, stream=stream, cone_max=cmax)
                        a1.record(stream)
                        stream.synchronize()
                        ts.append(a0.elapsed_time(a1))
                        cone.append(GG.last_forward_stats() / gg.num_pins)
                    row[mode] = {"ms_median": float(np.median(ts[1:] if len(ts) > 1 else ts)),
                                 "ms_mean": float(np.mean(ts)), "pins_recomputed_frac": float(np.median(cone))}
                out[f"{frac:g}"] = row
        return out

    # reverse-cone incremental backward: after each cone pass, insta_backward_update
    # on the kept gradient vs a full insta_backward into another buffer (bit-identical results; CUDA events)
    def bwd_series(GG, gg, fracs_steps, seed0):
        out = {}
        H = GG.schedule()["num_heads"]
        dk = torch.zeros((gg.num_arcs, 2), dtype=torch.float32, device=dev)
        df = torch.empty_like(dk)
        with torch.cuda.stream(stream):
            GG.forward(3.0, 0.0, 0, stream=stream)
            GG.backward_update(dk, stream=stream)
            for frac, nst in fracs_steps:
                tu, tf, hr, same = [], [], [], True
                for k in range(nst):
                    ids, m, sg = (torch.as_tensor(x, device=dev) for x in synth.sizing_step(gg, seed0 + k, frac=frac))
                    GG.update_arcs(ids, m, sg, incremental=True, stream=stream)
                    GG.forward(3.0, 0.0, 0, sync=False, stream=stream, cone_max=10 ** 12)
                    e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
                    e[0].record(stream)
                    inc = GG.backward_update(dk, stream=stream)   # default policy (full past E/5e4 arcs)
                    e[1].record(stream)
                    GG.backward(out=df, stream=stream)
                    e[2].record(stream)
                    stream.synchronize()
                    tu.append(e[0].elapsed_time(e[1]))
                    tf.append(e[1].elapsed_time(e[2]))
                    hr.append(GG.last_backward_stats() / H if inc else 1.0)
                    same = same and bool(torch.equal(dk.view(torch.int32), df.view(torch.int32)))
                out[f"{frac:g}"] = {"arcs_per_step": int(round(frac * gg.num_arcs)) or 1, "steps": nst,
                                    "update_ms_median": float(np.median(tu[1:])), "full_ms_median": float(np.median(tf[1:])),
                                    "heads_rerun_frac": float(np.median(hr)), "incremental_steps": int(sum(x < 1.0 for x in hr)),
                                    "bit_identical": same}
        return out

    incremental = None
    if args.incremental and world == 1:
        big = 10 ** 12
        c4 = inc_series(G, g, [(1e-7, 20), (1e-5, 20), (1e-4, 10)], [("incremental", 0), ("full", 0)], 7000)
        incremental = {"C4_small_updates": c4,
                       "what": "per step: insta_update_arcs + insta_forward (CUDA events); incremental = default "
                               "policy (cone pass for <= max(64, E/5e4) updated arcs), full = the same updates "
                               "then a full pass"}
        incremental["C4_backward_update"] = bwd_series(G, g, [(1e-7, 12), (1e-6, 12), (1e-5, 12), (1e-4, 8)], 8000)
        incremental["C4_backward_update_what"] = (
            "per step: a 1-cell .. 1e-4 sizing update + cone forward (untimed), then insta_backward_update on the "
            "kept TNS gradient (reverse cone; update_ms) vs insta_backward into another buffer (full_ms), CUDA "
            "events; heads_rerun_frac = work heads whose Eq 6 chain was re-run")
        try:
            g3 = synth.generate("C3")
            G3 = insta.Graph(g3, device=local)
            c3 = inc_series(G3, g3, [(0.01, args.c3_steps)],
                            [("incremental", 0), ("cone_forced", big), ("full", 0)], 3030)
            G3.close()
            row = c3["0.01"]
            incremental["C3_1pct_steps"] = row
            incremental["C3_speedup_vs_full"] = {m: row["full"]["ms_median"] / row[m]["ms_median"]
                                                 for m in ("incremental", "cone_forced")}
        except Exception as ex:  # pragma: no cover
            incremental["C3_1pct_steps"] = f"failed: {ex}"

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cores, model = host_info()
        try:
            gg = g if args.cpu_full else None
            npins, dt = cpu_oracle_sample(args.config, args.ref_sample_pins, args.tau, omp=False, g=gg)
            npo, dto = cpu_oracle_sample(args.config, args.ref_sample_pins, args.tau, omp=True, g=gg)
            what = "the full workload" if args.cpu_full else f"a {npins}-pin sample of the {cfg.name} recipe"
            cpu = {"value": npins / dt, "unit": UNIT, "cores": 1, "kind": "oracle", "cpu_model": model,
                   "host_cores": cores,
                   "sample": f"{what} ({npins} pins), fp64 fwd+slack+bwd, 1 run, 1 thread",
                   "all_cores": {"value": npo / dto, "unit": UNIT, "cores": cores,
                                 "what": "OpenMP level-parallel build of the same oracle (pins of a level in "
                                         "parallel), all cores in the affinity mask, 1 run"}}
        except Exception as ex:  # pragma: no cover
            cpu = {"value": None, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": f"failed: {ex}"}

    launches_per_step = 4 if args.schedule in (0, 2, 3) else 2 * G.num_levels + 2
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{cfg.name}: synthetic 3nm-shaped timing graph, {N} pins, {E} arcs, "
                                   f"{P} endpoints, {G.num_levels} levels",
                       "pins": N, "arcs": E, "endpoints": P, "levels": G.num_levels, "tau": args.tau,
                       "n_sigma": 3.0, "schedule": {0: "entry-parallel dataflow sweep forward + sweep backward", 1: "per-level",
                                                    2: "dataflow forward + dataflow backward",
                                                    3: "entry-parallel sweep forward (level barriers) + sweep backward"}[args.schedule],
                       "super_levels": sched["num_super_levels"], "folded_pins": sched["num_folded"],
                       "parallelism": f"replicas x{world}",
                       "l2": "working set > 126 MB L2 (no flush between passes; the `cold` leg flushes)",
                       "tns": s.tns, "wns": s.wns, "violations": s.num_violations,
                       "precision": "fp32 inputs, fp64 mean/variance state, fp32 sqrt/exp, fp64 TNS"},
            "fwd_ms": fwd_ms, "bwd_ms": bwd_ms, "fwd_bwd_ms": ms_step,
            "fwd_pins_per_s": N / (fwd_ms * 1e-3),
            "roofline": roofline, "lse": lse_leg, "cold": cold,
            "cpu_baseline": cpu, "e2e": e2e, "e2e_incremental": e2e_inc, "clocks": clk, "gpu_launches": launches_per_step * args.steps,
            "batched": batched, "topk": topk, "topk_wide": topk_wide, "clark": clark, "place": place, "incremental": incremental,
            "paper_context": "PAPER.md L9/L37: full-graph propagation < 0.1 s on a 15M-pin 3nm design, 1x A100 "
                             "(forward only, Top-K not stated); not the same metric",
        }
        print(json.dumps(line), flush=True)
    G.close()
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
