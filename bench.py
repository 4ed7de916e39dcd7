#!/usr/bin/env python3
"""bench.py -- all-pairs 1024-bit GCD throughput of libbulkgcd on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Workload (BASELINE.json metric "1024-bit GCDs/sec (all-pairs)", configs[2]):
all 134,209,536 pairs (i < j) of 16,384 synthetic 1024-bit RSA moduli with 8
planted shared primes (synth.config_moduli(3), seed 2018) -- the paper's
Table V workload size.  One step = one full pass of the hot
path: blocked layout of the resident moduli (H1), the all-pairs band kernel
(H2-H9) and, for N > 1, the NCCL all-gather of the hit lists; N GPUs split the
cohort range into balanced row bands (strong scaling: total work fixed).

value   : device-timed (CUDA events, sum over the K steps, max over ranks),
          moduli resident in HBM; L2 flushed (256 MiB write) before each step.
e2e     : the same metric through the public API with HOST buffers: N = 1:
          bulkgcd_all_pairs() (C ABI: H2D, kernels, D2H, sort); N > 1:
          dist.all_pairs_distributed() per rank.  Host-timed per call.
roofline: the hot kernel, integer-issue bound ("alu"):
          algorithmic integer lane-ops per launch (4 per limb-step + 16 per
          iteration, counted exactly by the kernel's stats pass on the same
          input) over its CUDA-event duration, against P_int = SMs x 4 SMSPs x
          32 lanes x 1 instruction/clk x the max SM clock of MEASURED_PEAKS.json;
          "alu_pipe" repeats it for the ALU-pipe share against the measured
          ALU-pipe rate (profiles/r1_pipemix.json); "traffic" is the ncu DRAM
          bytes per launch of the same build (profiles/r2_ncu_traffic.json).
cpu_baseline (rank 0, N = 1): the C oracle (Original Euclid, oracle/) on a
          bounded seeded sample of the same pairs, all host cores.
--impl reference: the oracle as it stands is the reference arm (no reference
          implementation exists; /root/reference is a paper).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# The paper's GTX 780 Ti, early-terminate, all pairs of 16K moduli (Table V):
# 0.346 us/GCD at 1024 bits, 1.33 us/GCD at 2048 bits.  Same workload size as cfg3 / cfg4.
PAPER_GCD_PER_S = {("cfg3", 1024): 1.0 / 0.346e-6, ("cfg4", 2048): 1.0 / 1.33e-6, ("cfg6", 512): 1.0 / 0.0773e-6}
METRIC = "1024-bit GCDs/sec (all-pairs)"
WORKLOADS = {
    "cfg1": "cfg1: all-pairs 1024-bit RSA moduli, n=64 (2,016 pairs), 3 planted shared primes (BASELINE.json configs[0])",
    "cfg3": "cfg3: all-pairs 1024-bit RSA moduli, n=16384 (134,209,536 pairs), 8 planted shared primes "
            "(BASELINE.json configs[2])",
    "cfg4": "cfg4: all-pairs 2048-bit RSA moduli, n=16384 (134,209,536 pairs), 8 planted shared primes "
            "(BASELINE.json configs[3])",
    "cfg5": "cfg5: all-pairs 1024-bit RSA moduli, n=65536 (2,147,450,880 pairs), 33 planted shared primes "
            "(BASELINE.json configs[4])",
    "cfg6": "cfg6: all-pairs 512-bit RSA moduli, n=16384 (134,209,536 pairs), 8 planted shared primes "
            "(the paper's 512-bit Table V workload; SURVEY.md §8(f) N1, not a BASELINE.json config)",
    "cfg7": "cfg7: all-pairs 4096-bit RSA moduli, n=512 (130,816 pairs), 4 planted shared primes "
            "(shared-memory kernels; SURVEY.md §8(f) N1, not a BASELINE.json config)",
    "cfg8": "cfg8: all-pairs 4096-bit moduli, n=16384 (134,209,536 pairs: the paper's Table V 4096-bit size, "
            "PAPER.md L451/L493), 8 planted shared factors; n = p*q from random odd 2048-bit cofactors "
            "(SURVEY.md §8(f) N1, not a BASELINE.json config)",
    "cfg2": "cfg2: 2^20 independent 1024-bit pair GCDs, exact mode (bulkgcd_pairs; the first 2^20 pairs i<j "
            "of a 1,449-moduli pool with 2 planted shared primes; BASELINE.json configs[1])",
}
UNIT = "GCD/s"
OPS_PER_LIMB, OPS_PER_ITER = 4, 16  # SURVEY.md §8(d) M2; DESIGN.md §Roofline
ALU_OPS_PER_LIMB = 3  # of the 4: IADD3, IADD3.X, SHF.R.W (ALU pipe); IMAD.WIDE.U32 is on the FMA pipe
PAPER_E_US = {512: 9.40, 1024: 28.6, 2048: 96.4, 4096: 357.0}  # Table V CPU (E), early-terminate, Xeon X7460 (L485-L493)


BACKEND = os.environ.get("BULKGCD_BENCH_BACKEND", "nccl")  # "gloo": test mode, ranks may share one GPU


def _coll(fn, *tensors, **kw):
    """Run a torch.distributed collective; with gloo, on host copies of device tensors."""
    if BACKEND != "gloo":
        return fn(*tensors, **kw)
    host = [t.cpu() for t in tensors]
    fn(*host, **kw)
    for t, h in zip(tensors, host):
        t.copy_(h)


def _allgather_into(out, inp):
    import torch.distributed as dist
    if BACKEND != "gloo":
        return dist.all_gather_into_tensor(out, inp)
    parts = [inp.new_empty(inp.shape).cpu() for _ in range(dist.get_world_size())]
    dist.all_gather(parts, inp.cpu())
    out.copy_(__import__("torch").cat(parts))


def _env_rank():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"sm_max_mhz": 1965.0}, "fallback"


def _alu_rate():
    """Measured ALU-pipe issue rate on this pool's B200s, warp-instructions/clk/SM:
    SHF.R.W alone (tools/pipemix.cu -> profiles/r1_pipemix.json; tools/pipemix2.cu
    -> profiles/r2_pipemix2.json re-measures 2.04 SMSP-cycles per SHF = 1.96/clk/SM)."""
    try:
        with open(os.path.join(ROOT, "profiles", "r1_pipemix.json")) as f:
            return float(json.load(f)["rates"]["SHF"]), "measured (profiles/r1_pipemix.json, SHF.R.W alone)"
    except (OSError, ValueError, KeyError):
        return 2.0, "guide unit counts (16 ALU lanes per SMSP)"


# ops_alg = 4 L + 16 I.  Of the 4 per limb-step, 3 are ALU-pipe (IADD3 / IADD3.X
# carry chains and the SHF.R.W funnel) and 1 (IMAD.WIDE.U32) FMA-heavy; of the 16 per iteration we
# count 8 as ALU-pipe (top-word fetch 2, compare 2, alpha select / parity 2, vote + branch 2) and 8
# as FP64 / XU / FMA work (reciprocal seed, Newton steps, quotient, conversions) -- DESIGN.md §7.
ALU_OPS_PER_ITER = 8


def roofline(limbs, iters, n_gcd, kern_s, sms, kernel, share, traffic, eff=None):
    """Roofline of the Euclid kernel.

    Bound "alu": integer issue.  achieved = algorithmic integer lane-ops per launch,
    ops_alg = 4 L + 16 I (M2; L = limb-steps, I = iterations, counted exactly by the
    kernel's stats pass on the same input), over the kernel's CUDA-event duration;
    peak P_int = SMs x 4 SMSPs x 32 lanes x 1 instruction/clk x the max SM clock
    (MEASURED_PEAKS.json sm_max_mhz; the guide's dispatch width: MEASURED_PEAKS has
    no integer peak).  Secondary "alu_pipe": the ALU-pipe share of ops_alg
    (3 L + 8 I) against the measured ALU-pipe rate.  `eff`: SIMT efficiencies from
    the stats pass (lane = useful lane-iterations / lane-slots; pass-word = limb-steps
    / words the warp's passes covered)."""
    peaks, src = _peaks()
    f = float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
    alu_ipc, alu_src = _alu_rate()
    ops = OPS_PER_LIMB * limbs + OPS_PER_ITER * iters
    alu_ops = ALU_OPS_PER_LIMB * limbs + ALU_OPS_PER_ITER * iters
    p_int = sms * 4 * 32 * f
    p_alu = sms * 32 * alu_ipc * f
    out = {"bound": "alu", "achieved": ops / kern_s / 1e12, "peak": p_int / 1e12, "unit": "T int lane-ops/s",
           "frac": ops / kern_s / p_int, "traffic": traffic, "kernel": kernel, "kernel_ms": kern_s * 1e3,
           "kernel_share_of_step": share, "ops_per_gcd": ops / n_gcd,
           "limb_steps_per_gcd": limbs / n_gcd, "iterations_per_gcd": iters / n_gcd,
           "peak_source": (f"P_int = {sms} SMs x 4 SMSPs x 32 lanes x 1 warp-instr/clk x {f / 1e6:.0f} MHz "
                           f"({src} MEASURED_PEAKS sm_max_mhz; SURVEY.md §8(d) M3, guide dispatch width)"),
           "alu_pipe": {"achieved": alu_ops / kern_s / 1e12, "peak": p_alu / 1e12, "frac": alu_ops / kern_s / p_alu,
                        "unit": "T ALU-pipe lane-ops/s", "ops_per_gcd": alu_ops / n_gcd,
                        "peak_source": f"ALU pipe {alu_ipc:.3f} warp-instr/clk/SM ({alu_src}) x 32 x {sms} x "
                                       f"{f / 1e6:.0f} MHz"}}
    if eff:
        out.update(eff)
    return out


def _traffic(workload: str):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of the workload's hot kernel,
    from the committed ncu --set full summary of the current build
    (profiles/r2_ncu_traffic.json, written by tools/ncu_traffic.py); None if absent."""
    try:
        with open(os.path.join(ROOT, "profiles", "r2_ncu_traffic.json")) as f:
            return json.load(f).get(workload, {}).get("dram_bytes_per_launch")
    except (OSError, ValueError):
        return None


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML while the timed region runs."""

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:  # no NVML: report what we have
            self.nv = None

    def _run(self):
        nv = self.nv
        names = {
            "hw_slowdown": getattr(nv, "nvmlClocksThrottleReasonHwSlowdown", 0x8),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksThrottleReasonSwThermalSlowdown", 0x20),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksThrottleReasonHwThermalSlowdown", 0x40),
            "sw_power_cap": getattr(nv, "nvmlClocksThrottleReasonSwPowerCap", 0x4),
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for k, bit in names.items():
                    if r & bit:
                        self.reasons.add(k)
            except Exception:
                pass
            self._stop.wait(0.05)

    def __enter__(self):
        if self.nv is not None:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv is not None:
            self.t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


REF_CALL_PAIRS = 1 << 18  # pairs per oracle call, shared by cpu_baseline and the --impl reference arm


def _sample_pairs(rng, m: int, k: int):
    """k seeded random pairs (i < j) of an m-moduli all-pairs workload."""
    i = rng.integers(0, m, size=2 * k + 64)
    j = rng.integers(0, m, size=2 * k + 64)
    keep = i < j
    return i[keep][:k], j[keep][:k]


def cpu_baseline(ms, target_s: float = 10.0, seed: int = 7):
    """The oracle (oracle/gcd_oracle.c, as it stands: classical Euclid + Knuth D) on a
    bounded seeded sample of the workload's pairs, all host cores, in calls of
    REF_CALL_PAIRS pairs (the reference arm's step), plus two single-core figures: the
    oracle, and the paper's own algorithm in C (oracle/approx_euclid.c, early-terminate:
    the analogue of Table V's CPU (E) column)."""
    import oracle
    cores = os.cpu_count() or 1
    rng = np.random.default_rng(seed)
    n_tot, dt = 0, 0.0
    while dt < target_s and n_tot < (1 << 23):
        i, j = _sample_pairs(rng, ms.m, REF_CALL_PAIRS)
        t0 = time.perf_counter()
        oracle.gcd_index_pairs(ms.N, i, j, nthreads=cores)
        dt += time.perf_counter() - t0
        n_tot += i.size
    i1, j1 = _sample_pairs(rng, ms.m, 1 << 13)  # one core, for the per-core figure
    t1 = time.perf_counter()
    oracle.gcd_index_pairs(ms.N, i1, j1, nthreads=1)
    dt1 = time.perf_counter() - t1
    # (E) on one core: calibrate, then ~4 s
    ie, je = _sample_pairs(rng, ms.m, 1 << 11)
    t2 = time.perf_counter()
    oracle.approx_index_pairs(ms.N, ie, je, ms.bits, True, nthreads=1)
    k = int(min(1 << 20, max(1 << 11, (1 << 11) / (time.perf_counter() - t2) * 4.0)))
    ie, je = _sample_pairs(rng, ms.m, k)
    t2 = time.perf_counter()
    _, _, ctr = oracle.approx_index_pairs(ms.N, ie, je, ms.bits, True, nthreads=1)
    dte = time.perf_counter() - t2
    return {"value": n_tot / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "value_1core": i1.size / dt1, "us_per_gcd_1core": dt1 / i1.size * 1e6,
            "sample": f"{n_tot} seeded random (i<j) pairs of the {ms.m}-moduli workload in calls of "
                      f"{REF_CALL_PAIRS}, exact classical Euclid (Knuth D) + the O3 map, {dt:.1f}s on {cores} threads; "
                      f"1-core figure on {i1.size} pairs",
            "paper_algorithm_E_1core": {
                "value": ie.size / dte, "unit": UNIT, "cores": 1, "us_per_gcd": dte / ie.size * 1e6,
                "iterations_per_gcd": ctr[0] / ie.size, "kind": "approximate-euclid (oracle/approx_euclid.c)",
                "paper_us_per_gcd": PAPER_E_US.get(ms.bits), "paper_hardware": "Xeon X7460, 1 thread (Table V, L491)",
                "sample": f"{ie.size} seeded random (i<j) pairs, early-terminate, {dte:.1f}s on 1 thread"}}


def run_reference(args):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only)."""
    rank, world, _ = _env_rank()
    if rank != 0:
        return
    import synth
    import oracle
    ms = synth.config_moduli(3)
    cores = os.cpu_count() or 1
    per_step = REF_CALL_PAIRS
    rng = np.random.default_rng(11)

    def step():
        i, j = _sample_pairs(rng, ms.m, per_step)
        t0 = time.perf_counter()
        G = oracle.gcd_index_pairs(ms.N, i, j, nthreads=cores)
        dt = time.perf_counter() - t0
        oracle.rsa_hit(oracle.bitlen_rows(G), 1024)
        return i.size, dt

    for _ in range(args.warmup):
        step()
    n_tot, t_tot = 0, 0.0
    for _ in range(args.steps):
        n, dt = step()
        n_tot += n
        t_tot += dt
    v = n_tot / t_tot
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_tot / args.steps * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": v / PAPER_GCD_PER_S[("cfg3", 1024)], "dtype": "u32", "data": "synthetic",
        "config": {"workload": "cfg3: all-pairs 1024-bit RSA moduli, n=16384 (134,209,536 pairs), 8 planted",
                   "per_step_sample_pairs": per_step, "mode": "rsa-early-terminate (oracle: exact gcd + O3 map)"},
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"{per_step} seeded random (i<j) pairs per step, exact classical Euclid"},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line))


def run_pairs(args):
    """cfg2 (BASELINE.json configs[1]): bulk execution of 2^20 independent exact
    GCDs through bulkgcd_pairs.  One step = word-interleave A and B (H1), the
    pairs kernel (exact mode, L41 + L107 to Y = 0) and the de-interleave of G.
    N > 1: contiguous chunks of the pairs per rank, no data-path collective
    ("replicas only" shape); total work fixed -> strong."""
    import torch
    import torch.distributed as dist

    import synth
    import paper_conf_ipps_fujitani15_b200 as bg

    rank, world, local = _env_rank()
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world} (launch N>1 with torchrun)")
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("gloo" if BACKEND == "gloo" else "nccl",
                                **({} if BACKEND == "gloo" else {"device_id": dev}))
    bg.bulkgcd_device_check()
    bits, W = 1024, 32
    A, B, pool = synth.config2()
    m_all = A.shape[0]
    lo, hi = m_all * rank // world, m_all * (rank + 1) // world
    A, B = np.ascontiguousarray(A[lo:hi]), np.ascontiguousarray(B[lo:hi])
    m = A.shape[0]
    m_pad = (m + 31) // 32 * 32
    dA = torch.from_numpy(A.view(np.int32)).to(dev)
    dB = torch.from_numpy(B.view(np.int32)).to(dev)
    dAc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dBc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dGc = torch.empty(m_pad * W, dtype=torch.int32, device=dev)
    dG = torch.empty(m * W, dtype=torch.int32, device=dev)
    dS = torch.zeros(8, dtype=torch.int64, device=dev)
    k0 = torch.cuda.Event(enable_timing=True)
    k1 = torch.cuda.Event(enable_timing=True)

    def step(flags=0):
        bg.bulkgcd_interleave(dA, dAc, m, m_pad, bits, True)
        bg.bulkgcd_interleave(dB, dBc, m, m_pad, bits, True)
        k0.record()
        bg.bulkgcd_pairs_device(dAc, dBc, dGc, m, m_pad, bits, bg.MODE_EXACT, None, dS, flags)
        k1.record()
        bg.bulkgcd_interleave(dGc, dG, m, m_pad, bits, False)

    step(bg.FLAG_STATS)  # algorithmic work (untimed stats pass)
    torch.cuda.synchronize()
    ctr = dS.cpu().numpy().astype(np.int64)
    iters, limbs, slots, passw = int(ctr[2]), int(ctr[4]), int(ctr[5]), int(ctr[6])
    eff = {"lane_efficiency": iters / slots if slots else None, "pass_word_efficiency": limbs / passw if passw else None}
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms, kern_ms = [], []
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            step()
            e1.record()
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
            kern_ms.append(k0.elapsed_time(k1))
    # correctness (outside the timed region): every result of this rank's chunk against the
    # construction ground truth of the pool (a planted prime for planted pairs, else 1)
    G = dG.cpu().numpy().view(np.uint32).reshape(m, W)
    want = np.zeros((m_all, W), np.uint32)
    want[:, 0] = 1
    npool = pool.m
    for a, b, g in pool.truth:
        k = a * npool - a * (a + 1) // 2 + (b - a - 1)  # row-major (i < j) position = cfg2 pair index
        if k < m_all:
            want[k] = synth.from_int(g, W)
    ok = bool(np.array_equal(G, want[lo:hi]))
    tot = torch.tensor([sum(step_ms), sum(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, tot, op=dist.ReduceOp.MAX)
    step_total_ms, kern_total_ms = float(tot[0]), float(tot[1])
    # e2e: bulkgcd_pairs with host buffers (H2D of A, B; D2H of G inside the call)
    e2e = []
    # the public path with PINNED host buffers (inputs and result), as an application would stage them
    pin = lambda a: torch.from_numpy(a.view(np.int32)).pin_memory().numpy().view(np.uint32)
    A, B = pin(A), pin(B)
    Gh = torch.empty(A.shape, dtype=torch.int32).pin_memory().numpy().view(np.uint32)
    if args.e2e_steps:  # one untimed warm-up call of the public path
        bg.bulkgcd_pairs(A, B, bits, out=Gh)
    for _ in range(args.e2e_steps):
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        bg.bulkgcd_pairs(A, B, bits, out=Gh)
        e2e.append(time.perf_counter() - t0)
    e2e_t = torch.tensor([sum(e2e)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, e2e_t, op=dist.ReduceOp.MAX)
    if rank == 0:
        value = m_all / (step_total_ms / 1e3 / args.steps)
        sms = torch.cuda.get_device_properties(dev).multi_processor_count
        kern_s = kern_total_ms / 1e3 / args.steps
        line = {
            "metric": "1024-bit GCDs/sec (bulk pairs, exact)", "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_total_ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": WORKLOADS["cfg2"], "pairs": m_all, "bits": bits, "mode": "exact",
                       "parallelism": f"contiguous chunks x{world} (no collective)",
                       "l2": "inputs larger than L2 (2 x 128 MiB operands + 128 MiB result)",
                       "ns_per_gcd": step_total_ms / args.steps * 1e6 / m_all,
                       "iterations_per_gcd": iters / m, "limb_steps_per_gcd": limbs / m,
                       "truth_ok": ok, "checked": int(m)},
            "roofline": dict(roofline(limbs, iters, m, kern_s, sms, f"pairs_kernel<{W}, exact>",
                                      kern_total_ms / step_total_ms, _traffic("cfg2"), eff),
                             hbm_bytes_per_gcd_alg=3 * W * 4, hbm_GBps_alg=3 * W * 4 * m / kern_s / 1e9),
            "e2e": {"value": m_all / (float(e2e_t[0]) / args.e2e_steps), "unit": UNIT,
                    "h2d_bytes_per_step": int(A.nbytes + B.nbytes) * world, "d2h_bytes_per_step": int(A.nbytes) * world},
            "gpu_launches": 4 * args.steps,
            "clocks": clk.summary(),
        }
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline_pairs(A, B)
        print(json.dumps(line))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def cpu_baseline_pairs(A, B, target_s: float = 10.0):
    """The oracle (exact classical Euclid) on a bounded prefix of the cfg2 pairs, all host cores."""
    import oracle
    cores = os.cpu_count() or 1
    k = 1 << 12
    t0 = time.perf_counter()
    oracle.gcd_batch(A[:k], B[:k], nthreads=cores)
    rate = k / (time.perf_counter() - t0)
    k = int(min(A.shape[0], max(1 << 14, rate * target_s)))
    t0 = time.perf_counter()
    oracle.gcd_batch(A[:k], B[:k], nthreads=cores)
    dt = time.perf_counter() - t0
    return {"value": k / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"the first {k} of the 2^20 cfg2 pairs, exact classical Euclid (Knuth D), {dt:.1f}s on "
                      f"{cores} threads"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--workload", default="cfg3", choices=sorted(WORKLOADS))
    ap.add_argument("--algo", default="E", choices=["E", "D", "C"],
                    help="all-pairs ablation (SURVEY.md §8(f) N2): E = Approximate Euclid (the product), "
                         "D = Fast Binary, C = Binary Euclid (the paper's Table V columns)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.workload == "cfg2":
        return run_pairs(args)

    import torch
    import torch.distributed as dist

    import synth
    import paper_conf_ipps_fujitani15_b200 as bg
    from paper_conf_ipps_fujitani15_b200 import dist as bgd

    rank, world, local = _env_rank()
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world} (launch N>1 with torchrun)")
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm = None
    if world > 1:
        if BACKEND == "gloo":
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
        comm = {"backend": dist.get_backend(), "rank": dist.get_rank(), "world": dist.get_world_size(),
                "device": f"cuda:{local}"}
        if BACKEND != "gloo":
            comm["nccl_version"] = ".".join(str(x) for x in torch.cuda.nccl.version())
        print(f"[bench] rank {comm['rank']}/{comm['world']} backend={comm['backend']} device={comm['device']}",
              file=sys.stderr, flush=True)
    bg.bulkgcd_device_check()

    # ---- inputs: rank 0 generates the seeded moduli, NCCL broadcast to the others
    k = int(args.workload[3:])
    cfgk = synth.CONFIG8 if k == 8 else synth.CONFIGS[k]
    bits = cfgk["bits"]
    W = bits // 32
    metric = f"{bits}-bit GCDs/sec (all-pairs)"
    if rank == 0:
        ms = synth.config_moduli(k)
        N = ms.N
        truth = ms.truth
    else:
        N = np.zeros((cfgk["m"], W), np.uint32)
        truth = None
    if world > 1:
        t = torch.from_numpy(N.view(np.int32)).to(dev)
        _coll(dist.broadcast, t, src=0)
        N = t.cpu().numpy().view(np.uint32)
    n = N.shape[0]
    pairs = n * (n - 1) // 2

    runner = bgd.AllPairsBand(N, bits, rank, world, device=dev)
    runner.upload(non_blocking=False)
    flush = torch.empty(64 << 20, dtype=torch.int32, device=dev)  # 256 MiB > 126 MB L2
    cap = runner.cap
    gbuf = torch.empty(world * cap * (2 + W), dtype=torch.int32, device=dev)
    gcnt = torch.empty(world, dtype=torch.int64, device=dev)

    algo_flag = {"E": 0, "D": bg.FLAG_ALGO_FAST_BINARY, "C": bg.FLAG_ALGO_BINARY}[args.algo]

    def step():
        runner.layout()
        k0.record()
        runner.search(algo_flag)
        k1.record()
        if world > 1:
            # the exchange step: NCCL all-gather of the hit counts and fixed-capacity hit buffers
            _allgather_into(gcnt, runner.d_ctr[:1])
            _allgather_into(gbuf, runner.d_hits)

    # ---- algorithmic work of one launch (stats pass, untimed)
    runner.layout()
    runner.search(bg.FLAG_STATS | algo_flag)
    torch.cuda.synchronize()
    ctr = runner.d_ctr.cpu().numpy().astype(np.int64)
    iters, limbs, slots, passw, betapos = int(ctr[2]), int(ctr[4]), int(ctr[5]), int(ctr[6]), int(ctr[7])
    if world > 1:
        tt = torch.tensor([iters, limbs, slots, passw, betapos], dtype=torch.int64, device=dev)
        _coll(dist.all_reduce, tt)
        iters, limbs, slots, passw, betapos = (int(x) for x in tt)
    # SIMT efficiencies of the lockstep register kernels (the smem kernels run lanes independently)
    eff = {"lane_efficiency": iters / slots if slots else None,
           "pass_word_efficiency": limbs / passw if passw else None} if args.algo == "E" else None

    k0 = torch.cuda.Event(enable_timing=True)
    k1 = torch.cuda.Event(enable_timing=True)
    for _ in range(args.warmup):
        flush.fill_(1)
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    step_ms, kern_ms = [], []
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t_wall = time.perf_counter()
        for _ in range(args.steps):
            flush.fill_(2)
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            step()
            e1.record()
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
            kern_ms.append(k0.elapsed_time(k1))
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t_wall = time.perf_counter() - t_wall

    # correctness of the timed steps' output (outside the timed region)
    local_hits = runner.local_hits()
    if world > 1:
        allrec = bgd.gather_hits(local_hits)
    else:
        allrec = local_hits
    found = bgd.records_to_hits(allrec.cpu().numpy(), bits).as_list()
    if rank != 0:
        ok = True
    elif k == 8:  # cofactor moduli: the planted pairs, each g a >= bits/2-bit common divisor (exact division)
        Ni = [synth.to_int(r) for r in N]
        ok = [(i, j) for i, j, _ in found] == [(a, b) for a, b, _ in truth] and all(
            g.bit_length() >= bits // 2 and Ni[i] % g == 0 and Ni[j] % g == 0 for i, j, g in found)
    else:
        ok = found == truth

    tot_ms = torch.tensor([sum(step_ms), sum(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, tot_ms, op=dist.ReduceOp.MAX)
    step_total_ms, kern_total_ms = float(tot_ms[0]), float(tot_ms[1])

    # ---- end to end through the public API with host buffers
    e2e_ms = []
    Nh = np.ascontiguousarray(N)
    d2h = 0
    if args.algo != "E":
        args.e2e_steps = 0  # the public API runs (E); an ablation has no end-to-end line
    if args.e2e_steps:  # one untimed warm-up call of the public path (allocator pools, lazy module loading)
        bg.bulkgcd_all_pairs(Nh, bits) if world == 1 else bgd.all_pairs_distributed(Nh, bits)
    for _ in range(args.e2e_steps):
        flush.fill_(3)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        if world == 1:
            h = bg.bulkgcd_all_pairs(Nh, bits)
        else:
            h = bgd.all_pairs_distributed(Nh, bits)
        dt = time.perf_counter() - t0
        d2h = 8 + h.ij.shape[0] * (2 + W) * 4
        e2e_ms.append(dt * 1e3)
    e2e_t = torch.tensor([sum(e2e_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        _coll(dist.all_reduce, e2e_t, op=dist.ReduceOp.MAX)
    e2e_value = pairs / (float(e2e_t[0]) / 1e3 / args.e2e_steps) if args.e2e_steps else None

    if rank == 0:
        value = pairs / (step_total_ms / 1e3 / args.steps)
        sms = torch.cuda.get_device_properties(dev).multi_processor_count
        kern_s = kern_total_ms / 1e3 / args.steps
        paper = PAPER_GCD_PER_S.get((args.workload, bits))
        line = {
            "metric": metric, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": step_total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": value / paper if paper else None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": WORKLOADS[args.workload],
                       "n": n, "bits": bits, "pairs": pairs, "mode": "rsa-early-terminate",
                       "algorithm": {"E": "approximate-euclid (" + ("register-resident" if W < 128 else
                                                                     "hybrid: one operand in registers, one in shared memory") + ")",
                                     "D": "fast-binary-euclid (ablation, smem)",
                                     "C": "binary-euclid (ablation, smem)"}[args.algo],
                       "parallelism": f"row-band x{world}" + (" + NCCL hit all-gather" if world > 1 else ""),
                       "l2": "flushed before every step (256 MiB write); inputs 2 MiB",
                       "ns_per_gcd": step_total_ms / args.steps * 1e6 / pairs,
                       "iterations_per_gcd": iters / pairs, "limb_steps_per_gcd": limbs / pairs,

                       "ms_per_step_median": statistics.median(step_ms), "ms_per_step_min": min(step_ms),
                       "hits_ok": bool(ok), "hits": len(found), "wall_s": t_wall},
            # per-GPU kernel throughput: each rank runs 1/world of the work
            "roofline": roofline(limbs / world, iters / world, pairs / world, kern_s, sms,
                                 (f"allpairs_kernel<{W}>" if W < 128 else f"allpairs_hybrid_kernel<{W}>")
                                 if args.algo == "E" else f"allpairs_*_kernel<{W}, {args.algo}>",
                                 kern_total_ms / step_total_ms,
                                 _traffic(args.workload) if args.algo == "E" else None, eff),
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(Nh.nbytes) * world,
                    "d2h_bytes_per_step": int(d2h) * world} if e2e_value else None,
            "gpu_launches": 2 * args.steps,
            "clocks": clk.summary(),
        }
        if comm:
            line["config"]["comm"] = comm
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(ms)
        print(json.dumps(line))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
