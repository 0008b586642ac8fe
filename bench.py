#!/usr/bin/env python
"""Benchmark of the DDA equation-solving hot path on B200 (BASELINE.json metric).

One STEP = one pass of the whole hot path on device-resident synthetic input:
  dda_build_matrix   (A1: springs -> upper-symmetric BSR6 + transpose map)
  dda_bj_setup       (A3: 6x6 Cholesky inverses)
  dda_pcg_solve      (A4-A6: block-Jacobi PCG to 1e-10, cold start d0 = 0;
                      one persistent kernel: symmetric SpMV + fused vector ops)
on the configs[4] workload at N=1: a ~1M-block jittered-brick slope (6M DOF),
which fits one B200 (the matrix is 1.29 GB).  `value` = device ms per step
(CUDA events on the launching stream, max over ranks); lower is better.

Extra keys: `roofline` for the dominant kernel (the persistent PCG kernel,
algorithmic bytes per launch / its CUDA-event duration vs the measured HBM
copy peak), `spmv` (the standalone symmetric SpMV GB/s and % of HBM peak —
the first half of the metric), `e2e` (dda_solve_host_batch over the K steps
with pinned host buffers: every step's copies inside the timed region, step
k+1's H2D overlapping step k's solve; `single_call` = one synchronous
dda_solve_host per step), `cpu_baseline` (the oracle, one
core, on a bounded sample), `clocks` (NVML, sampled during the timed region).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference] [--blocks N]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np

METRIC = "BSR6 sym SpMV GB/s & % HBM peak; PCG solve ms to 1e-10 at 1/2/4/8 B200"
UNIT = "ms"
DEFAULT_BLOCKS = 1_000_000


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def traffic_for(n_blocks: int, which: str):
    """DRAM bytes per launch from the committed ncu --set full capture of the same
    workload (profiles/traffic.json), or None."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(p) as f:
            t = json.load(f)
        if int(t.get("n_blocks", -1)) != n_blocks:
            return None
        e = t[which]
        return {"bytes": e["traffic_bytes_per_launch"], "source": e["source"]}
    except Exception:
        return None


def l2_roofline(n_blocks: int, iters: int, pcg_ms: float):
    """The secondary (L2) roofline of the PCG loop: its L2 sector traffic per iteration from the committed
    ncu capture of k_sp_loop (profiles/traffic.json "sp_loop_l2"), times the iterations of this solve,
    over the solve's CUDA-event time, against the practical L2 (LTS) throughput cap of the
    microarchitecture guide (~6.3 kB per SM-clock cycle at the SM clock of the capture)."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        e = t["sp_loop_l2"]
        if int(t.get("n_blocks", -1)) != n_blocks:
            return None
    except Exception:
        return None
    tbps = e["l2_bytes_per_iter"] * iters / (pcg_ms * 1e-3) / 1e12
    cap = e["lts_cap_bytes_per_cycle"] * e["sm_clock_hz"] / 1e12
    out = {"l2_bytes_per_iter": e["l2_bytes_per_iter"], "achieved_tbps": tbps, "cap_tbps": cap,
           "frac": tbps / cap, "source": e["source"]}
    if "note" in e:
        out["note"] = e["note"]
    return out


def bytes_per_row_spmv(u: float) -> float:
    """Algorithmic bytes of one symmetric SpMV per block row:
    D 288 + u*(V 288 + col 4 + low_row 4 + low_to_up 4) + row_ptr/low_ptr 8 + x 48 + y 48."""
    return 392.0 + 300.0 * u


def pcg_launch_bytes(n: int, u: float, iters: int) -> float:
    """Algorithmic bytes of one k_pcg launch with block-Jacobi, d0 = 0:
    init 432 B/row (F, Dinv read; d, r, z, p written); iteration 0: SpMV of p + phase B 528
    (p, d, r, q, Dinv read; d, r, z written); iterations k >= 1: SpMV whose x = z + beta p_old
    is two vectors (+48) and whose owner writes p_new (+48), + phase B 528; final
    true-residual SpMV + 96 (F, q read)."""
    S = bytes_per_row_spmv(u)
    it = max(iters, 1)
    return n * (432.0 + (S + 528.0) + (it - 1) * (S + 96.0 + 528.0) + S + 96.0)


def pcg_launch_bytes_scaled(n: int, nnzb: int, iters: int, checks: int) -> float:
    """Algorithmic bytes of one dda_pcg_solve on the scaled block-Jacobi engine, d0 = 0
    (DESIGN.md §6), per block row unless noted:
    k_scale_upper: nnzb*(288 V read + 288 written + 8 indices) + n*192 (S);
    k_s_init 384 (F, S read; r~, p, x written);
    iteration 0: scaled SpMV 300u + 8 + 96 (p read, q written) + phase B 152 (r~, q read; r~ written;
    the stopping-test weight w_i, 8 B);
    iterations k >= 1: the SpMV also reads p_old (+48), writes p (+48) and applies the deferred
    x += alpha p_old (x read + written, +96) + phase B 152;
    each exact stopping test (k_s_check, `checks` of them) 240 (r~ + L read);
    k_s_final 336 (x, p, S read; d written); the true-residual SpMV on K + 96 (F, q read)."""
    u = nnzb / n
    it = max(iters, 1)
    sp = 300.0 * u + 8.0 + 96.0
    return (nnzb * 584.0 + n * 192.0
            + n * (384.0 + (sp + 152.0) + (it - 1) * (sp + 192.0 + 152.0) + 240.0 * checks + 336.0
                   + bytes_per_row_spmv(u) + 96.0))


class ClockSampler:
    """NVML sampler of SM clock and throttle reasons during the timed region."""

    def __init__(self, index: int, period: float = 0.05):
        self.index, self.period = index, period
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        self.ok = False

    def __enter__(self):
        try:
            import pynvml as N
            N.nvmlInit()
            h = N.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM)
            names = {
                "gpu_idle": getattr(N, "nvmlClocksEventReasonGpuIdle", 0x1),
                "applications_clocks_setting": 0x2,
                "sw_power_cap": 0x4,
                "hw_slowdown": 0x8,
                "sync_boost": 0x10,
                "sw_thermal_slowdown": 0x20,
                "hw_thermal_slowdown": 0x40,
                "hw_power_brake_slowdown": 0x80,
                "display_clock_setting": 0x100,
            }

            def run():
                while not self._stop.is_set():
                    try:
                        self.samples.append(N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM))
                        fn = getattr(N, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                            N.nvmlDeviceGetCurrentClocksThrottleReasons
                        mask = fn(h)
                        for k, bit in names.items():
                            if mask & bit and k != "gpu_idle":
                                self.reasons.add(k)
                    except Exception:
                        pass
                    time.sleep(self.period)

            self._t = threading.Thread(target=run, daemon=True)
            self._t.start()
            self.ok = True
        except Exception as e:  # no NVML: report it rather than guess
            self.err = repr(e)
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["nvml_unavailable"]}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def dist_env():
    return int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0"))


# ----------------------------------------------------------------------------- CPU oracle legs

ORACLE_1M = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "r02_oracle_1m.json")


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_iters_for(P):
    """The oracle's own BJ-PCG iteration count to 1e-10 on this exact system, from the committed
    record of tools/oracle_1m.py (synth + oracle only; checked by problem fingerprint), or None."""
    try:
        rec = json.load(open(ORACLE_1M))
    except (OSError, ValueError):
        return None, None
    import hashlib
    h = hashlib.sha256()
    for a in (P.bi, P.bj, P.pen, P.F):
        h.update(np.ascontiguousarray(a).tobytes())
    if rec.get("n_blocks") != P.n or rec.get("fingerprint") != h.hexdigest()[:16]:
        return None, None
    return int(rec["oracle_iters"]), rec


def oracle_step_at_size(P, k_sample: int = 8, spmv_stats: dict = None):
    """The oracle (as it stands, one pinned host core) on THE WORKLOAD ITSELF, bounded by PCG
    iterations: assembly O-1 + expansion O-2 are timed whole; the PCG (block inverses, r0, the
    iterations, the true residual) is timed at maxit = 1 and at maxit = 1 + k_sample, which gives
    the per-iteration time; the step is assembly + PCG(1) + (I - 1) x per-iteration, with I the
    oracle's own iteration count on this system (tools/oracle_1m.py's committed full solve; if it
    is missing or stale the full solve runs here once).  Returns (ms, info dict)."""
    import oracle
    oracle.build()
    aff = os.sched_getaffinity(0)
    core = sorted(aff)[0]
    os.sched_setaffinity(0, {core})
    try:
        t0 = time.perf_counter()
        M = oracle.assemble(P)
        M.full_csr()
        t1 = time.perf_counter()
        M.pcg(P.F, tol=1e-300, maxit=1, precond="bj")
        t2 = time.perf_counter()
        M.pcg(P.F, tol=1e-300, maxit=1 + k_sample, precond="bj")
        t3 = time.perf_counter()
        iters, rec = oracle_iters_for(P)
        src = "profiles/r02_oracle_1m.json (tools/oracle_1m.py: the oracle's full solve of this system)"
        if iters is None:
            _, iters, _, _ = M.pcg(P.F, tol=1e-10, maxit=10000, precond="bj")
            src = "the oracle's full solve, run here"
        if spmv_stats is not None:
            x = np.random.default_rng(7).uniform(-1.0, 1.0, 6 * P.n)
            one = []
            for _ in range(3):
                a = time.perf_counter(); M.spmv(x); one.append(time.perf_counter() - a)
            spmv_stats["spmv_1_thread_ms"] = 1000.0 * statistics.median(one)
    finally:
        os.sched_setaffinity(0, aff)
    if spmv_stats is not None:
        os.sched_setaffinity(0, aff)
        x = np.random.default_rng(7).uniform(-1.0, 1.0, 6 * P.n)
        par, th = [], 1
        for _ in range(3):
            a = time.perf_counter(); _, th = M.spmv_par(x); par.append(time.perf_counter() - a)
        spmv_stats.update({"spmv_all_cores_ms": 1000.0 * statistics.median(par), "all_cores_threads": th})
    per_it = (t3 - t2) / k_sample
    ms = 1000.0 * ((t1 - t0) + (t2 - t1) + (iters - 1) * per_it)
    info = {"assemble_expand_ms": 1000.0 * (t1 - t0), "pcg_1_iter_ms": 1000.0 * (t2 - t1),
            "per_iter_ms": 1000.0 * per_it, "iters": iters, "iters_source": src, "k_sample": k_sample,
            "measured_s": t3 - t0, "pinned_core": core, "cpu_model": cpu_model()}
    return ms, info


def oracle_sample_text(P, info):
    return (f"the oracle on the workload itself ({P.n} blocks), one pinned core ({info['cpu_model']}): "
            f"assembly+expansion {info['assemble_expand_ms']:.0f} ms and BJ-PCG (block inverses, r0, 1 "
            f"iteration, true residual) {info['pcg_1_iter_ms']:.0f} ms measured whole; PCG iterations "
            f"measured over {info['k_sample']} ({info['per_iter_ms']:.1f} ms each) and counted at the "
            f"oracle's own {info['iters']} iterations to 1e-10 ({info['iters_source']}); no block-count "
            f"scaling; {info['measured_s']:.1f} s of CPU time measured")


def run_reference(args):
    """--impl reference: the oracle timed as it stands on the host cores (rank 0 only)."""
    world, rank, _ = dist_env()
    if rank != 0:
        return
    from synth import make_slope, preset
    P = make_slope(preset(args.blocks, seed=1005))
    for _ in range(args.warmup):
        oracle_step_at_size(P, k_sample=2)
    times, info = [], None
    for _ in range(args.steps):
        ms, info = oracle_step_at_size(P, k_sample=args.ref_iter_sample)
        times.append(ms)
    ms = statistics.median(times)
    sample = oracle_sample_text(P, info)
    line = {"impl": "reference", "metric": METRIC, "value": ms, "unit": UNIT, "higher_is_better": False,
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(args.blocks), "n_blocks": P.n,
                       "sample": f"PCG iterations sampled: {info['k_sample']} of {info['iters']} per step"},
            "cpu_baseline": {"value": ms, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             "cpu_model": info["cpu_model"]},
            "e2e": {"value": ms, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_name(n):
    return (f"slope-{n // 1000}k: jittered-brick slope (configs[4] at N=1), ~{n} blocks = {6 * n} DOF, "
            f"~5 contacts/block; assemble + BJ setup + BJ-PCG to 1e-10 (cold start)")


# ----------------------------------------------------------------------------- our arm

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--blocks", type=int, default=DEFAULT_BLOCKS)
    ap.add_argument("--precond", default="bj")
    ap.add_argument("--spmv-reps", type=int, default=20)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-iter-sample", type=int, default=8, help="oracle PCG iterations timed (cpu_baseline)")
    ap.add_argument("--ref-iter-sample", type=int, default=4, help="oracle PCG iterations timed per reference step")
    ap.add_argument("--clock-period", type=float, default=0.05, help="NVML clock sampling period (s)")
    ap.add_argument("--dist-transport", default="ipc", choices=["ipc", "nccl"],
                    help="N > 1: peers' buffers mapped with CUDA IPC handles, one persistent kernel per rank (v7; "
                         "falls back to nccl if the mapping fails) or NCCL halo + allreduce per iteration (v4)")
    ap.add_argument("--force-dist", action="store_true",
                    help="run the partitioned (NCCL) path even at N = 1 (a check of the N > 1 code path)")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
        return

    import torch
    world, rank, local = dist_env()
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            raise SystemExit("launch N>1 with torchrun (one process per GPU)")
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import __graft_entry__
    __graft_entry__.build() if rank == 0 else None
    if world > 1:
        torch.distributed.barrier()
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    from synth import make_slope, preset

    P = make_slope(preset(args.blocks, seed=1005))
    if world > 1 or args.force_dist:
        if world == 1:
            import torch.distributed as dist
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", "29511")
            dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", local))
        run_dist(args, P, world, rank, local)
        return
    t = dda.problem_to_device(P)
    stream = torch.cuda.current_stream()
    hbm_peak, peak_src = measured_peaks()

    def step(ev=None):
        if ev: ev[0].record(stream)
        K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
        if ev: ev[1].record(stream)
        K.bj_setup()
        if ev: ev[2].record(stream)
        d, it, rr, st = K.pcg_solve(t["F"], tol=1e-10, maxit=10000, precond=args.precond)
        if ev: ev[3].record(stream)
        return K, d, it, rr, st

    engine = None
    for _ in range(args.warmup):
        K, d, it, rr, st = step()
        engine = K.pcg_engine(args.precond)
        checks = K.last_checks()
        K.free()
    torch.cuda.synchronize()

    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(args.steps)]
    start, stop = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    results = []
    l0 = dda.launch_count()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local, args.clock_period) as clk:
        start.record(stream)
        for k in range(args.steps):
            K, d, it, rr, st = step(evs[k])
            results.append((K.n, K.nnzb, it, rr, st))
            K.free()
        stop.record(stream)
        torch.cuda.synchronize()
    launches = dda.launch_count() - l0
    total_ms = start.elapsed_time(stop)
    ms_step = total_ms / args.steps
    if world > 1:
        tt = torch.tensor([ms_step], device="cuda")
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        ms_step = float(tt.item())
    ph_build = statistics.median(e[0].elapsed_time(e[1]) for e in evs)
    ph_bj = statistics.median(e[1].elapsed_time(e[2]) for e in evs)
    ph_pcg = [e[2].elapsed_time(e[3]) for e in evs]
    n, nnzb, iters, rel_res, status = results[-1]
    assert all(r[4] == dda.OK for r in results), results
    assert rel_res <= 1e-10 * 1.01, rel_res
    u = nnzb / n
    pcg_ms = statistics.mean(ph_pcg)
    if engine == "scaled" and dda.lib().dda__get_scaled_loop() == 1:
        engine = "scaled_persistent"
        pcg_bytes = pcg_launch_bytes_scaled(n, nnzb, iters, checks)
        pcg_kernel = ("dda_pcg_solve, scaled block-Jacobi engine: k_scale_upper (S_i V_ij S_j^T) + k_s_init + ONE "
                      "persistent cooperative kernel k_sp_loop running every iteration (phase A fused p-update + "
                      "SpMV + x update, phase B r~ update, rare phase C exact stopping test; grid barriers) + "
                      f"k_s_final + true-residual SpMV; {checks} exact stopping tests")
    elif engine == "scaled":
        pcg_bytes = pcg_launch_bytes_scaled(n, nnzb, iters, checks)
        pcg_kernel = ("dda_pcg_solve, scaled block-Jacobi engine: k_scale_upper (S_i V_ij S_j^T) + one CUDA-graph "
                      "while loop (k_g_spmv<SC> + k_s_update + k_s_check per iteration) with its prelude/epilogue "
                      f"kernels; {checks} exact stopping tests")
    else:
        pcg_bytes = pcg_launch_bytes(n, u, iters)
        pcg_kernel = ("dda_pcg_solve: one CUDA-graph while loop (k_g_spmv + k_g_update per iteration) with its "
                      "prelude/epilogue kernels")
    ach = pcg_bytes / (pcg_ms * 1e-3) / 1e9

    # ---- standalone symmetric SpMV (metric's first half), back to back (hot, as PCG sees it)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    x = torch.rand(6 * n, dtype=torch.float64, device="cuda") * 2 - 1
    y = torch.empty_like(x)
    for _ in range(3):
        K.spmv(x, y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(args.spmv_reps):
        K.spmv(x, y)
    e1.record(stream)
    torch.cuda.synchronize()
    spmv_ms = e0.elapsed_time(e1) / args.spmv_reps
    spmv_bytes = n * bytes_per_row_spmv(u)
    spmv_gbs = spmv_bytes / (spmv_ms * 1e-3) / 1e9
    K.free()
    del x, y

    # ---- e2e: the host-buffer C ABI, pinned host buffers, H2D + D2H of every step inside the timed region.
    # Headline: dda_solve_host_batch over K steps (system k+1's host->device copy and system k's
    # device->host copy overlap system k's assembly + solve; per step = total / K).  Also reported: one
    # synchronous dda_solve_host call per step (no cross-step overlap).
    e2e = None
    if not args.no_e2e:
        pin = lambda a: torch.from_numpy(a).pin_memory()
        hk, hbi, hbj, hpen, he, hg, hF = (pin(P.kdiag), pin(P.bi), pin(P.bj), pin(P.pen), pin(P.e), pin(P.g), pin(P.F))
        K_e2e = max(1, args.steps)
        hds = [torch.empty(6 * n, dtype=torch.float64).pin_memory() for _ in range(K_e2e)]
        hd = hds[0]
        dda.solve_host(hk, hbi, hbj, hpen, he, hg, hF, out=hd.numpy())   # warm
        torch.cuda.synchronize()
        single_ms = []
        for _ in range(max(1, min(args.steps, 3))):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            _, it2, rr2, st2 = dda.solve_host(hk, hbi, hbj, hpen, he, hg, hF, out=hd.numpy())
            a1.record(stream)
            torch.cuda.synchronize()
            single_ms.append(a0.elapsed_time(a1))
        systems = [dict(kdiag=hk, bi=hbi, bj=hbj, pen=hpen, e=he, g=hg, F=hF, d=hds[k]) for k in range(K_e2e)]
        dda.solve_host_batch(systems[:2])   # warm (the two input slots' allocation is then cached)
        torch.cuda.synchronize()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        res = dda.solve_host_batch(systems)
        a1.record(stream)
        torch.cuda.synchronize()
        batch_ms = a0.elapsed_time(a1) / K_e2e
        assert all(r[2] == dda.OK for r in res), res
        assert all(torch.equal(hds[k], hds[0]) for k in range(1, K_e2e))
        h2d = sum(a.numel() * a.element_size() for a in (hk, hbi, hbj, hpen, he, hg, hF))
        e2e = {"value": batch_ms, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(hd.numel() * 8), "steps": K_e2e,
               "api": "dda_solve_host_batch (C ABI, pinned host buffers; step k+1's H2D and step k's D2H overlap "
                      "step k's assembly + solve)",
               "single_call": {"value": statistics.median(single_ms), "unit": UNIT,
                               "api": "dda_solve_host (C ABI, one synchronous call per step)"}}

    # ---- CPU oracle baseline (rank 0, N=1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        sst = {}
        ms_cpu, info = oracle_step_at_size(P, k_sample=args.cpu_iter_sample, spmv_stats=sst)
        cpu = {"value": ms_cpu, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": oracle_sample_text(P, info),
               "cpu_model": info["cpu_model"], "host_cores": os.cpu_count(),
               "spmv_oracle": {"one_thread_ms": sst.get("spmv_1_thread_ms", 0.0),
                               "all_cores_ms": sst.get("spmv_all_cores_ms", 0.0),
                               "all_cores_threads": sst.get("all_cores_threads", 1),
                               "note": ("one oracle SpMV (full scalar CSR, O-3) on the workload, 1 pinned thread "
                                        "and the OpenMP all-cores twin (labelled second number, SURVEY §8(d)); "
                                        "the GPU SpMV is the line's spmv.ms")}}

    line = {
        "metric": METRIC, "value": ms_step, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": False, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(args.blocks), "n_blocks": n, "dof": 6 * n, "springs": P.m,
                   "contacts": P.n_contacts, "nnzb_upper": nnzb, "u": round(u, 3), "precond": args.precond,
                   "tol": 1e-10, "start": "cold (d0 = 0)",
                   "l2": f"inputs larger than L2 (matrix {(n * 288 + nnzb * 300) / 1e9:.2f} GB vs 126 MB L2); no flush",
                   "parallelism": f"dp{world}" if world > 1 else "single GPU",
                   "step": "dda_build_matrix + dda_bj_setup + dda_pcg_solve"},
        "phases_ms": {"assemble": ph_build, "bj_setup": ph_bj, "pcg": pcg_ms, "pcg_iters": iters,
                      "pcg_us_per_iter": 1000.0 * pcg_ms / max(iters, 1), "true_rel_res": rel_res},
        "roofline": {"kernel": pcg_kernel, "engine": engine,
                     "bound": "hbm", "achieved": ach, "peak": hbm_peak, "unit": "GB/s", "frac": ach / hbm_peak,
                     "traffic": traffic_for(n, "pcg_" + str(engine)), "peak_source": peak_src,
                     "algorithmic_bytes_per_launch": pcg_bytes, "l2": l2_roofline(n, iters, pcg_ms)},
        "spmv": {"kernel": "k_spmv3<FULL,3,5> (column-pair map, two blocks in flight per lane, 3 CTAs/SM)", "ms": spmv_ms, "traffic": traffic_for(n, "spmv"), "gbs": spmv_gbs, "frac_hbm": spmv_gbs / hbm_peak,
                 "gflops": n * (72 + 144 * u) / (spmv_ms * 1e-3) / 1e9, "bytes": spmv_bytes,
                 "timing": "back to back (hot), inputs > L2"},
        "e2e": e2e, "cpu_baseline": cpu, "gpu_launches": int(launches),
        "clocks": clk.summary(),
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def run_dist(args, P, world, rank, local):
    """N > 1: block-row partitioned BJ-PCG over NCCL.  One step per
    rank = assemble the local matrix (springs touching own rows) + distributed
    PCG to 1e-10; value = max over ranks of the device time."""
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    bounds = dda.row_bounds(P.n, world)
    r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
    n_own = r1 - r0
    # every rank gets the global spring list; dda_build_matrix_dist selects the springs of its rows
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    t = {k: dev(getattr(P, k)) for k in ("bi", "bj", "pen", "e", "g")}
    t["kdiag"] = dev(P.kdiag[r0:r1])
    t["F"] = dev(P.F[6 * r0:6 * r1])
    transport = args.dist_transport
    comm = None
    if transport == "ipc":
        # v7 over CUDA IPC: build this rank's partition, exchange the handle blobs over the process group,
        # map the peers (every later rebuild re-attaches into the mapped buffers)
        try:
            comm = dda.Comm.ipc(world, rank)
            comm.build_matrix_dist(0, P.n, bounds, t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
            blobs = [None] * world
            dist.all_gather_object(blobs, comm.ipc_export())
            comm.ipc_import(blobs)
            ok = torch.tensor([1], device="cuda")
        except Exception as exc:   # noqa: BLE001 -- every rank must agree on the fallback
            print(f"ipc transport unavailable ({exc}); falling back to nccl", file=sys.stderr)
            ok = torch.tensor([0], device="cuda")
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if int(ok.item()) == 0:
            if comm is not None:
                comm.free()
            comm, transport = None, "nccl"
    if comm is None:
        obj = [dda.Comm.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        comm = dda.Comm.nccl(world, rank, obj[0])
    stream = torch.cuda.current_stream()
    hbm_peak, peak_src = measured_peaks()

    def step(ev=None):
        if ev: ev[0].record(stream)
        K = comm.build_matrix_dist(0, P.n, bounds, t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
        if ev: ev[1].record(stream)
        ds, it, rr, st = comm.pcg_solve([t["F"]], tol=1e-10, maxit=10000, precond=args.precond)
        if ev: ev[2].record(stream)
        return K, it, rr, st

    if transport == "ipc":   # a failed IPC solve (e.g. a bounded wait expired) falls back to NCCL on every rank
        try:
            _, _, _, st0 = step()
            ok = torch.tensor([1 if st0 == dda.OK else 0], device="cuda")
        except Exception as exc:   # noqa: BLE001
            print(f"ipc solve failed ({exc}); falling back to nccl", file=sys.stderr)
            ok = torch.tensor([0], device="cuda")
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if int(ok.item()) == 0:
            comm.free()
            obj = [dda.Comm.unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            comm, transport = dda.Comm.nccl(world, rank, obj[0]), "nccl"
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    start, stop = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = dda.launch_count()
    dist.barrier()
    torch.cuda.synchronize()
    res = []
    with ClockSampler(local, args.clock_period) as clk:
        start.record(stream)
        for k in range(args.steps):
            res.append(step(evs[k]))
        stop.record(stream)
        torch.cuda.synchronize()
    dist.barrier()
    launches = dda.launch_count() - l0
    ms = start.elapsed_time(stop) / args.steps
    asm = statistics.median(e[0].elapsed_time(e[1]) for e in evs)
    pcg = statistics.mean(e[1].elapsed_time(e[2]) for e in evs)
    K, iters, rel_res, status = res[-1]
    assert status == dda.OK and rel_res <= 1.01e-10, (status, rel_res)
    # algorithmic bytes per own row and iteration: v4 (NCCL) 300u + 496 (phase A 300u + 152,
    # phase B 344); v7 (IPC) the single-GPU scaled engine's 300u + 448; u over the rank's own rows
    info = comm.info(0, nparts=world)
    u = K.nnzb / max(n_own, 1)
    local_bytes = n_own * (300.0 * u + (448.0 if transport == "ipc" else 496.0)) * iters
    ach = local_bytes / (pcg * 1e-3) / 1e9
    tt = torch.tensor([ms, pcg, asm], device="cuda")
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    ms, pcg_max, asm_max = (float(v) for v in tt.tolist())
    # comm / compute split: one extra (untimed) solve with CUDA events between the steps of every
    # iteration (halo exchange, phase A, allreduce, phase B; DDA_DIST_PROFILE=1), max over ranks
    import ctypes as _C
    if transport == "nccl":
        os.environ["DDA_DIST_PROFILE"] = "1"
        comm.pcg_solve([t["F"]], tol=1e-10, maxit=10000, precond=args.precond)
        os.environ.pop("DDA_DIST_PROFILE")
        prof = (_C.c_double * 4)()
        fprof = dda.lib().dda__dist_profile
        fprof.argtypes = [_C.c_void_p, _C.c_void_p]
        fprof(comm._h, prof)
        tp = torch.tensor(list(prof), device="cuda")
        dist.all_reduce(tp, op=dist.ReduceOp.MAX)
        split = {"halo_ms": float(tp[0]), "phaseA_ms": float(tp[1]), "allreduce_ms": float(tp[2]),
                 "phaseB_ms": float(tp[3]), "note": "per solve, summed over iterations, max over ranks; one "
                                                    "profiled (event-instrumented, untimed) solve"}
    else:
        split = {"note": "v7 over CUDA IPC: one persistent kernel per rank, halo reads and the one-shot allreduce "
                         "inside it; no per-phase host events"}
    # e2e: pinned host local inputs -> device, assemble, solve, d -> host (max over ranks)
    e2e = None
    if not args.no_e2e:
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
        h = {k: pin(getattr(P, k)) for k in ("bi", "bj", "pen", "e", "g")}
        h["kdiag"] = pin(P.kdiag[r0:r1])
        h["F"] = pin(P.F[6 * r0:6 * r1])
        hd = torch.empty(6 * n_own, dtype=torch.float64).pin_memory()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        dist.barrier()
        a0.record(stream)
        dd = {k: v.cuda(non_blocking=True) for k, v in h.items()}
        K2 = comm.build_matrix_dist(0, P.n, bounds, dd["kdiag"], dd["bi"], dd["bj"], dd["pen"], dd["e"], dd["g"])
        ds, _, _, _ = comm.pcg_solve([dd["F"]], tol=1e-10, precond=args.precond)
        hd.copy_(ds[0], non_blocking=True)
        a1.record(stream)
        torch.cuda.synchronize()
        e2 = torch.tensor([a0.elapsed_time(a1)], device="cuda")
        dist.all_reduce(e2, op=dist.ReduceOp.MAX)
        h2d = sum(v.numel() * v.element_size() for v in h.values())
        e2e = {"value": float(e2.item()), "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(hd.numel() * 8),
               "api": "dda_build_matrix_dist + dda_pcg_solve_dist (per-rank pinned host inputs: the global springs, "
                      "own diagonal terms and F)"}
    if rank == 0:
        line = {
            "metric": METRIC, "value": ms, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(args.blocks), "n_blocks": P.n, "dof": 6 * P.n, "springs": P.m,
                       "precond": args.precond, "tol": 1e-10, "start": "cold (d0 = 0)",
                       "parallelism": (f"block-row partition over {world} ranks, one persistent kernel per rank, "
                                       "peers' buffers mapped with CUDA IPC (halo reads and one-shot allreduce "
                                       "over NVLink)" if transport == "ipc" else
                                       f"block-row partition over {world} ranks (NCCL halo + allreduce)"),
                       "transport": transport,
                       "rank0_rows": n_own, "rank0_halo": info["n_halo"],
                       "step": "dda_build_matrix_dist (select + renumber + assemble + plan, device) + "
                               "dda_pcg_solve_dist",
                       "l2": "inputs larger than L2 per rank at 1M/N; no flush"},
            "phases_ms": {"assemble_max": asm_max, "pcg_max": pcg_max, "pcg_iters": iters,
                          "pcg_us_per_iter": 1000.0 * pcg_max / max(iters, 1), "true_rel_res": rel_res,
                          "comm_compute_split": split},
            "roofline": {"kernel": "rank 0: dist v4 scaled engine (k_v4_a Ks SpMV + sigma / r~.q / q.q, k_v4_b "
                                   "r~, p, x updates + stopping sums; one NCCL halo of p and one 6-double "
                                   "allreduce per iteration)",
                         "bound": "hbm",
                         "achieved": ach, "peak": hbm_peak, "unit": "GB/s", "frac": ach / hbm_peak,
                         "traffic": None, "peak_source": peak_src, "per": "GPU (rank 0)"},
            "e2e": e2e, "cpu_baseline": None, "gpu_launches": int(launches), "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    comm.free()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
