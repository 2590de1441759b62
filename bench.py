#!/usr/bin/env python
"""Benchmark: sparse-grid evaluations/sec at d=10, n=11 (127,574,017 surpluses).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl sg|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...          (N > 1)

One step = one pass of the whole hot path over one batch:
  a7  compression: rank 0 copies the nodal values of function A into the
      surplus buffer and hierarchizes it (sg_hierarchize);
  e   N > 1: one NCCL broadcast of the 1.02 GB surplus array (the only
      collective of the path);
  a1-a6 decompression: every rank orders the whole 10^7-query batch along one
      global Morton curve (sg_sfc_order, deterministic) and evaluates the
      rank's contiguous range of that order (sg_evaluate_ordered).
Strong scaling (default): ONE batch of 10^7 queries split over
the ranks; --scaling weak gives every rank its own 10^7-query batch.
`value` = evaluations of the batch / max-over-ranks step time.
`e2e`   = the same step through the public API (Grid.hierarchize_ +
          multi.evaluate_distributed) with the nodal values and queries copied
          from pinned host memory and the results copied back inside the
          timed region.
`roofline` = the evaluation kernel (the dominant one), timed with CUDA events
          on its launching stream inside the library (sg_profile_*).
`cpu_baseline` = the C oracle (oracle/) on a bounded sample of the same
          queries on all host cores (rank 0, N = 1 only).

--impl reference runs the oracle itself as the reference arm (this tier has
no reference implementation to install).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import sginputs as S  # noqa: E402

CFG = S.CONFIGS["cfg3"]
METRIC = "sparse-grid evaluations/sec at d=10,n=11 (127M pts), 1/2/4/8 B200"
UNIT = "evals/s"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


def workload_config(m_batch, n_gpus, weak=False):
    split = ("1e7 queries per GPU (rows [rank*1e7, (rank+1)*1e7) of the SplitMix64 stream, seed 0x5EED0003), "
             "each rank's batch Morton-ordered on its GPU" if weak else
             "one batch of 1e7 uniform random queries (SplitMix64 stream, seed 0x5EED0003) held by every rank, "
             "ordered along one global Morton curve (sg_sfc_order, identical on every rank), rank r evaluating "
             "the r-th contiguous range of that order (sg_evaluate_ordered)")
    return {"workload": "cfg3: d=10, n=11 sparse grid (127,574,017 fp64 surpluses, function A hierarchized on rank 0 "
                        "each step and broadcast), " + split,
            "d": CFG["d"], "n": CFG["n"], "num_points": 127574017,
            "queries_per_gpu": m_batch if weak else -(-m_batch // n_gpus),
            "global_batch": m_batch * n_gpus if weak else m_batch,
            "parallelism": f"query ranges x{n_gpus} of one global order, alpha broadcast" if not weak
            else f"independent batches x{n_gpus}, alpha broadcast",
            "l2": "inputs larger than L2 (1.02 GB surpluses, 0.8 GB queries); no flush"}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.path = None

    def start(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except FileNotFoundError:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        self.proc.wait()
        rows = []
        with open(self.path) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) >= 9:
                    rows.append(parts)
        os.unlink(self.path)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[5 + k].lower().startswith("active")})
        loaded = [s for s in sm if mx and s > 0.5 * max(mx)] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def oracle_sample(alpha_host, x_host, budget_s=15.0, max_q=20000):
    """Time the C oracle (as it stands) on a bounded prefix of the batch, all host cores."""
    import oracle
    d, n = CFG["d"], CFG["n"]
    cores = oracle.max_threads()
    k0 = max(cores, 16)
    t0 = time.perf_counter()
    y0, a0 = oracle.evaluate(d, n, alpha_host, x_host[:k0])
    t_cal = time.perf_counter() - t0
    k = int(min(max_q, max(k0, budget_s / max(t_cal, 1e-6) * k0)))
    k = max(cores, (k // cores) * cores)
    t0 = time.perf_counter()
    y, a = oracle.evaluate(d, n, alpha_host, x_host[:k])
    dt = time.perf_counter() - t0
    return k, dt, cores, y, a


# ------------------------------------------------------------------ reference arm
def run_reference(args, rank, world):
    if rank != 0:
        return
    import oracle
    oracle.build()
    d, n = CFG["d"], CFG["n"]
    N = oracle.num_points(d, n)
    # surpluses: closed form of function A's hierarchization would skip the
    # oracle's own compression; the reference arm times decompression on the
    # random-surplus source B (same evaluation cost per query).
    alpha = S.random_surplus(N, seed=CFG["seed"])
    cores = oracle.max_threads()
    per_step = max(cores, int(os.environ.get("SG_REF_QUERIES", 4 * cores)))
    x = S.queries(d, per_step * (args.steps + args.warmup), CFG["seed"])
    for w in range(args.warmup):
        oracle.evaluate(d, n, alpha, x[w * per_step:(w + 1) * per_step])
    t0 = time.perf_counter()
    for s in range(args.steps):
        a = (args.warmup + s) * per_step
        oracle.evaluate(d, n, alpha, x[a:a + per_step])
    dt = time.perf_counter() - t0
    value = per_step * args.steps / dt
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": workload_config(CFG["m"], world),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"{per_step} cfg3 queries per step (of the 1e7-query workload), "
                                       f"random surpluses, oracle/sg_oracle.c or_evaluate"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ product arm
def run_sg(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_murarasuwbbp11_b200 as P
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    d, n = CFG["d"], CFG["n"]
    weak = args.scaling == "weak"
    m_rank = args.m or CFG["m"]  # weak: queries per rank; strong: the whole batch
    m_batch = m_rank if weak else (args.m or CFG["m"])
    g = P.Grid(d, n)
    N = g.num_points

    # nodal values of function A at the grid points (input generation, untimed)
    values = torch.empty(N, dtype=torch.float64, device=dev)
    chunk = 1 << 23
    for a in range(0, N, chunk):
        b = min(N, a + chunk)
        values[a:b] = S.f_A_torch(g.coords(a, b - a, device=dev))
    alpha = torch.empty_like(values)
    # strong: every rank holds the whole seeded batch (rows 0..m-1) and evaluates its range of the one
    # global Morton order; weak: rank r's own batch is rows [r*m, (r+1)*m) of the stream
    x = S.queries_torch(d, m_batch, CFG["seed"], device=dev, first=rank * m_batch if weak else 0)
    y = torch.zeros(m_batch, dtype=torch.float64, device=dev)
    perm = torch.empty(m_batch, dtype=torch.int32, device=dev)
    ws = torch.empty(g.workspace_bytes(m_batch), dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    ev = {k: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for k in ("bcast", "order")}
    acc = {"bcast": 0.0, "order": 0.0}
    timing = {"on": False}

    def timed(k, fn):
        if not timing["on"]:
            return fn()
        ev[k][0].record(stream)
        r = fn()
        ev[k][1].record(stream)
        ev[k][1].synchronize()
        acc[k] += ev[k][0].elapsed_time(ev[k][1])
        return r

    def step():
        if rank == 0:
            alpha.copy_(values)
            g.hierarchize_(alpha)
        if world > 1:
            timed("bcast", lambda: multi.replicate_surpluses(alpha, src=0))  # the path's one collective
        timed("order", lambda: P.sg_sfc_order(g.handle, x, perm, ws))
        if weak:
            g.evaluate_ordered(alpha, x, perm, 0, m_batch, out=y)
        else:
            multi.evaluate_distributed(g, alpha, x, out=y, perm=perm, broadcast=False)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    for _ in range(args.warmup):
        step()
    barrier()
    P.sg_profile_read(reset=True)
    P.sg_profile_enable(True)
    clocks = ClockSampler(local_rank)
    if rank == 0:
        clocks.start()
    launches0 = P.sg_kernel_launch_count()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    barrier()
    elapsed_ms = max_over_ranks(ev0.elapsed_time(ev1))
    launches = P.sg_kernel_launch_count() - launches0
    prof = P.sg_profile_read(reset=True)
    P.sg_profile_enable(False)
    clk = clocks.stop() if rank == 0 else None
    ms_per_step = elapsed_ms / args.steps
    total_queries = m_batch * world if weak else m_batch
    value = total_queries / (ms_per_step / 1e3)
    first, count = (0, m_batch) if weak else multi.partition(m_batch, world, rank)

    # phase breakdown (separate untimed pass with per-phase events; max over ranks)
    timing["on"] = True
    step()
    timing["on"] = False
    bcast_ms = max_over_ranks(acc["bcast"])
    order_ms = max_over_ranks(acc["order"])
    eval_ms_rank = max_over_ranks(prof["eval_ms"] / max(1, args.steps))

    # ---- e2e through the public API: host buffers, copies inside the timed region
    e2e = None
    if not args.no_e2e:
        values_h = values.cpu().pin_memory() if rank == 0 else None
        x_h = x.cpu().pin_memory()
        y_h = torch.empty(m_batch, dtype=torch.float64, pin_memory=True)
        x_d = torch.empty_like(x)
        y_d = torch.zeros_like(y)

        def step_e2e():
            if rank == 0:
                alpha.copy_(values_h, non_blocking=True)
                g.hierarchize_(alpha)
            x_d.copy_(x_h, non_blocking=True)
            if weak:
                g.evaluate(alpha, x_d, out=y_d, workspace=ws)
            else:
                multi.evaluate_distributed(g, alpha, x_d, out=y_d, broadcast=world > 1)
            y_h.copy_(y_d, non_blocking=True)
            stream.synchronize()

        for _ in range(2):  # warm-up (the first timed step after a single warm-up step ran ~200 ms long)
            step_e2e()
        barrier()
        e2e_steps = max(1, min(args.steps, args.e2e_steps))
        evk = [torch.cuda.Event(enable_timing=True) for _ in range(e2e_steps + 1)]
        ev0.record(stream)
        evk[0].record(stream)
        for k in range(e2e_steps):
            step_e2e()
            evk[k + 1].record(stream)
        ev1.record(stream)
        barrier()
        e2e_ms = max_over_ranks(ev0.elapsed_time(ev1)) / e2e_steps
        e2e_step_ms = [evk[k].elapsed_time(evk[k + 1]) for k in range(e2e_steps)]
        # phase breakdown of one more e2e step (events on the stream; untimed)
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
        evs[0].record(stream)
        if rank == 0:
            alpha.copy_(values_h, non_blocking=True)
        evs[1].record(stream)
        if rank == 0:
            g.hierarchize_(alpha)
        x_d.copy_(x_h, non_blocking=True)
        evs[2].record(stream)
        if weak:
            g.evaluate(alpha, x_d, out=y_d, workspace=ws)
        else:
            multi.evaluate_distributed(g, alpha, x_d, out=y_d, broadcast=world > 1)
        evs[3].record(stream)
        y_h.copy_(y_d, non_blocking=True)
        evs[4].record(stream)
        stream.synchronize()
        e2e_phases = {"h2d_surplus_values": evs[0].elapsed_time(evs[1]),
                      "hierarchize_and_h2d_queries": evs[1].elapsed_time(evs[2]),
                      "order_and_evaluate": evs[2].elapsed_time(evs[3]), "d2h_results": evs[3].elapsed_time(evs[4])}
        own = perm[first:first + count].long().cpu()
        assert torch.equal(y_h[own], y.cpu()[own]), "e2e results differ from the device path"
        e2e = {"value": total_queries / (e2e_ms / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": (N * 8 if rank == 0 else 0) + m_batch * d * 8, "d2h_bytes_per_step": m_batch * 8,
               "ms_per_step": e2e_ms, "steps": e2e_steps, "step_ms_rank0": e2e_step_ms,
               "breakdown_ms_rank0": e2e_phases,
               "path": "Grid.hierarchize_ + multi.evaluate_distributed (sg_sfc_order + sg_evaluate_ordered) "
                       "between pinned-host copies" if not weak else "Grid.evaluate between pinned-host copies"}

    if rank != 0:
        return

    # ---- roofline of the evaluation kernel
    pk, pk_src = peaks()
    T = g.num_subspaces
    f_mhz = float(pk.get("sm_max_mhz", 1965.0))
    eval_ms = prof["eval_ms"] / max(1, prof["eval_launches"])  # per sg_evaluate_ordered call (rank 0)
    gathered = T * 8 * count  # one fp64 surplus per subspace per query of this rank's range
    achieved = gathered / (eval_ms / 1e3) / 1e9  # GB/s
    lsu_peak = 148 * 128 * f_mhz * 1e6 / 1e9  # L1/SMEM -> RF, 128 B/clk/SM
    fma = math.comb(n + d, d) - 1
    fp64_peak = 148 * 64 * 2 * f_mhz * 1e6 / 1e12  # TFLOP/s, 64 DFMA/clk/SM
    fp64_achieved = 2 * fma * count / (eval_ms / 1e3) / 1e12
    traffic = None
    prof_json = os.path.join(ROOT, "profiles", "eval_kernel_ncu.json")
    if os.path.exists(prof_json):
        with open(prof_json) as f:
            pj = json.load(f)
        if pj.get("m") == count and pj.get("d") == d and pj.get("n") == n:
            traffic = pj.get("dram_bytes_per_launch")
    roofline = {"bound": "alu", "pipe": "L1/LSU gather of surpluses (128 B/clk/SM x 148 SMs)",
                "achieved": achieved, "peak": lsu_peak, "unit": "GB/s", "frac": achieved / lsu_peak,
                "traffic": traffic, "peak_source": f"derived: 148 SMs x 128 B/clk x {f_mhz:.0f} MHz "
                                                  f"({pk_src} sm_max_mhz)",
                "kernel_ms": eval_ms, "algorithmic_bytes_per_launch": gathered,
                "fp64": {"achieved": fp64_achieved, "peak": fp64_peak, "unit": "TFLOP/s",
                         "frac": fp64_achieved / fp64_peak, "fma_per_eval": fma}}

    # ---- CPU baseline: the oracle on a bounded sample (rank 0, N = 1 only)
    cpu = None
    parity = None
    if world == 1 and not args.no_cpu:
        alpha_h = alpha.cpu().numpy()
        x_np = x[:20000].cpu().numpy()
        k, dt, cores, yo, ao = oracle_sample(alpha_h, x_np, budget_s=args.cpu_budget)
        cpu = {"value": k / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"first {k} of the 1e7 cfg3 queries ({dt:.1f} s), same surpluses"}
        err = np.abs(y[:k].cpu().numpy() - yo) / ao
        parity = {"queries_checked": k, "max_normwise_err": float(err.max()), "tol": 1e-12,
                  "pass": bool(err.max() <= 1e-12)}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak" if weak else "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": workload_config(m_batch, world, weak),
            "clocks": clk, "e2e": e2e, "gpu_launches": int(launches), "roofline": roofline,
            "cpu_baseline": cpu, "parity": parity,
            "breakdown_ms_per_step": {"evaluate_kernel_max_rank": eval_ms_rank,
                                      "sfc_order_max_rank": order_ms, "broadcast_max_rank": bcast_ms,
                                      "hierarchize_rank0": prof["hier_ms"] / max(1, args.steps),
                                      "hierarchized_points_per_s": N / (prof["hier_ms"] / max(1, args.steps) / 1e3)
                                      if prof["hier_ms"] > 0 else None,
                                      "value_excl_broadcast": total_queries / ((ms_per_step - bcast_ms) / 1e3)}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="sg", choices=["sg", "reference"])
    ap.add_argument("--m", type=int, default=0, help="queries (strong: the whole batch; weak: per GPU); default 1e7")
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="strong (default): one 1e7-query batch split over the GPUs by ranges of its global "
                         "Morton order; weak: a 1e7-query batch per GPU")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        run_sg(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
