"""bench.py — throughput of the distributed particle filter hot path on B200.

Metric (BASELINE.json): "state estimates/sec at 1M particles; particle-steps/sec
at 1/2/4/8 B200".  ``value`` is whole-job particle-steps/s; at N = 1 the
workload is config C2 (paper's medium arm, d = 9, 4096 sub-filters x 256 = 2^20
particles, ring t = 1, RWS) and ``estimates_per_s`` is its state-estimate rate.
At N > 1 (torchrun, one rank per GPU) each GPU holds 2^20 particles of ONE
filter of N x 2^20 particles with the cross-GPU halo exchange and the global
estimate reduce every step (weak scaling).

Timing: W warm-up steps, then K steps each bracketed by CUDA events on the
filter's stream, with an L2 flush (a 512 MiB write) between steps outside the
events; barrier + synchronize on both sides; max over ranks.  ``e2e`` is the
same metric through the C ABI with host inputs (pinned staging inside pf_step)
and a device->host estimate read every step.  ``--impl reference`` times the
CPU oracle (the only other place bench.py runs oracle/) on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

NJ, M_SUB, N_SUB, T_EX = 5, 256, 4096, 1          # config C2 per GPU
D = NJ + 4
PARTICLES_PER_GPU = M_SUB * N_SUB
METRIC = "state estimates/sec at 1M particles; particle-steps/sec at 1/2/4/8 B200"
DATA = ("synthetic: seeded lemniscate-tracking trajectory of the 5-joint arm (workload.py, reading R16); "
        "prior X0 ~ N(mu0, sigma0) drawn on device")


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="budget of the oracle cpu_baseline")
    ap.add_argument("--no-extras", action="store_true", help="skip the Vose / L2-resident extra timings")
    return ap.parse_args()


def _config(world: int) -> dict:
    return {"workload": "C2: medium robotic arm (n_joints 5, d 9), 1M particles per GPU",
            "n_joints": NJ, "m": M_SUB, "n_filters_per_gpu": N_SUB, "n_filters": N_SUB * world,
            "particles": PARTICLES_PER_GPU * world, "topology": "ring", "t": T_EX, "resampler": "rws",
            "l2": "flushed between timed steps (512 MiB write)", "parallelism": f"dp{world} (sub-filter shards)"}


def _oracle_rate(seconds: float, steps_cap: int | None = None, n_sample: int = 256):
    """Particle-steps/s of the CPU oracle (single thread) on a bounded sample
    of the C2 workload: n_sample sub-filters of 256 particles."""
    from oracle import orc
    from paper_conf_ipps_chitchianasks13_b200 import workload as W
    T = 400
    tr = W.make_trajectory(NJ, T, 0)
    f = orc.Filter(orc.Config(m=M_SUB, n_filters=n_sample, t=T_EX, topo="ring", resampler="rws", seed=1),
                   orc.Model(n_joints=NJ), tr["mu0"], tr["sigma0"])
    times = []
    t_all = time.perf_counter()
    k = 1
    while k <= T:
        t0 = time.perf_counter()
        f.step(tr["Z"][k], tr["U"][k - 1])
        f.estimate()
        times.append(time.perf_counter() - t0)
        k += 1
        if steps_cap is not None and len(times) >= steps_cap:
            break
        if steps_cap is None and time.perf_counter() - t_all > seconds:
            break
    particles = M_SUB * n_sample
    return particles * len(times) / sum(times), len(times), particles, times


def run_reference(a) -> None:
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    # warm-up steps untimed, then K timed steps, each a bounded sample of C2
    _oracle_rate(0, steps_cap=max(a.warmup, 1), n_sample=64)
    rate, nsteps, particles, times = _oracle_rate(0, steps_cap=a.steps, n_sample=64)
    sample = f"oracle (plain C, 1 thread) on 64 of the 4096 sub-filters x 256 of C2, {nsteps} steps"
    line = {"metric": METRIC, "value": rate, "unit": "particle-steps/s", "impl": "reference",
            "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * sum(times) / nsteps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": DATA,
            "config": _config(1), "estimates_per_s": rate / PARTICLES_PER_GPU,
            "cpu_baseline": {"value": rate, "unit": "particle-steps/s", "cores": 1, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": rate, "unit": "particle-steps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


class ClockSampler:
    """nvidia-smi-equivalent clock / throttle sampling (NVML) during a region."""

    def __init__(self, index: int):
        self.samples, self.reasons, self._stop = [], set(), threading.Event()
        self.active = False   # record only while a timed region runs
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
            self.max_mhz = None

    def _run(self):
        nv = self.nv
        names = {
            "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4, "hw_slowdown": 0x8,
            "sync_boost": 0x10, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
            "hw_power_brake_slowdown": 0x80, "display_clock_setting": 0x100}
        while not self._stop.is_set():
            if self.active:
                try:
                    self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                    self.reasons |= {k for k, b in names.items() if r & b and k != "gpu_idle"}
                except Exception:
                    pass
            time.sleep(0.002)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def run_ours(a) -> None:
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_chitchianasks13_b200 import distributed as Dd
    from paper_conf_ipps_chitchianasks13_b200 import filter as F
    from paper_conf_ipps_chitchianasks13_b200 import workload as W

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one rank per GPU over NCCL; with fewer visible GPUs than ranks (a
    # functional check of the multi-rank path on one device) ranks share GPUs
    # and the host-side plumbing runs over gloo
    shared = world > 1 and torch.cuda.device_count() < world
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    K, Wm = a.steps, max(a.warmup, 3)
    T = Wm + K + 8
    tr = W.make_trajectory(NJ, T, 0)
    N = N_SUB * world
    kw = dict(m=M_SUB, n_filters=N, t=T_EX, topo="ring", seed=2013, rank=rank, world=world)
    model = F.ArmModel(n_joints=NJ)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if shared else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    sampler = ClockSampler(local)
    sampler.__enter__()
    zs = torch.tensor(tr["Z"][1:], device=dev)
    us = torch.tensor(tr["U"][:-1], device=dev)

    transport = {"p2p": False}   # multi-rank: halo + estimate inside the kernel (peer transport) or NCCL

    # ---- device-resident inputs (value) -----------------------------------
    def device_run(resampler: str, flush_l2: bool, steps: int):
        pf = F.ParticleFilter(tr["mu0"], tr["sigma0"], model, resampler=resampler, device_inputs=True, **kw)
        df = Dd.DistributedFilter(pf)
        transport["p2p"] = df.p2p
        stream = pf.stream
        for k in range(Wm):
            df.step(zs[k], us[k])
        barrier()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        sampler.active = True
        if flush_l2:
            for i in range(steps):
                flush.zero_()
                ev[i][0].record(stream)
                df.step(zs[Wm + i], us[Wm + i])
                ev[i][1].record(stream)
        else:
            ev[0][0].record(stream)
            for i in range(steps):
                df.step(zs[Wm + i], us[Wm + i])
            ev[-1][1].record(stream)
        torch.cuda.synchronize()
        sampler.active = False
        barrier()
        if flush_l2:
            ms = sum(s.elapsed_time(e) for s, e in ev)
        else:
            ms = ev[0][0].elapsed_time(ev[-1][1])
        ms = max_over_ranks(ms)
        est = pf.estimate()
        pf.close()
        return ms / steps, est

    ms_step, est = device_run("rws", True, K)
    steps_per_s = 1e3 / ms_step
    value = steps_per_s * PARTICLES_PER_GPU * world

    extras = {}
    if not a.no_extras:
        ms_v, _ = device_run("vose", True, K)
        ms_w, _ = device_run("rws", False, K)
        extras = {"vose": {"estimates_per_s": 1e3 / ms_v, "ms_per_step": ms_v,
                           "particle_steps_per_s": 1e3 / ms_v * PARTICLES_PER_GPU * world},
                  "l2_resident": {"estimates_per_s": 1e3 / ms_w, "ms_per_step": ms_w,
                                  "note": "back-to-back steps, particle set (84 MB) left in the 126 MB L2"}}

    # ---- end to end through the C ABI with host buffers --------------------
    pf = F.ParticleFilter(tr["mu0"], tr["sigma0"], model, resampler="rws", **kw)
    df = Dd.DistributedFilter(pf)
    Zh = np.ascontiguousarray(tr["Z"][1:], np.float32)
    Uh = np.ascontiguousarray(tr["U"][:-1], np.float32)
    for k in range(Wm):
        df.step(Zh[k], Uh[k])
        df.estimate()
    barrier()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    sampler.active = True
    for i in range(K):
        flush.zero_()
        ev[i][0].record(pf.stream)
        df.step(Zh[Wm + i], Uh[Wm + i])        # H2D of z_k, u_{k-1} inside pf_step
        df.estimate()                          # D2H of the estimate record + sync
        ev[i][1].record(pf.stream)
    torch.cuda.synchronize()
    sampler.active = False
    sampler.__exit__()
    clocks = sampler.summary()
    barrier()
    e2e_ms = max_over_ranks(sum(s.elapsed_time(e) for s, e in ev) / K)
    pf.close()
    e2e_value = 1e3 / e2e_ms * PARTICLES_PER_GPU * world

    # ---- roofline of the step kernel ----------------------------------------
    # algorithmic bytes per launch: read + write the (d+1)
    # floats of every particle, write the best-t mailbox row of every
    # sub-filter, read deg*t mailbox entries per sub-filter (ring deg = 2)
    E = D + 2
    bytes_launch = PARTICLES_PER_GPU * 8 * (D + 1) + N_SUB * T_EX * E * 4 * (1 + 2)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = peaks.get("hbm_gbs", 6650.0)
    achieved = bytes_launch / (ms_step * 1e-3) / 1e9
    traffic, instr = None, None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))
        traffic = prof.get("C2", {}).get("dram_bytes_per_launch")
        instr = prof.get("C2", {}).get("lane_instr_per_particle")
    except Exception:
        pass
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": "pf_step_kernel", "bytes_per_launch": bytes_launch,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "fallback 6.65 TB/s",
                "note": "issue-bound: see roofline_issue and DESIGN.md §6"}
    # the binding roofline: instruction issue (148 SMs x 4 schedulers x 32 lanes
    # per clock at the sampled SM clock); executed lane-instructions per
    # particle-step from the committed ncu capture of this kernel at C2
    roofline_issue = None
    if instr:
        mhz = clocks.get("sm_mhz") or 1965
        peak_i = 148 * 4 * 32 * mhz * 1e6 / 1e12
        ach_i = instr * PARTICLES_PER_GPU / (ms_step * 1e-3) / 1e12
        roofline_issue = {"bound": "alu", "achieved": ach_i, "peak": peak_i, "unit": "T lane-instr/s",
                          "frac": ach_i / peak_i, "instr_per_particle": instr,
                          "source": "profiles/ncu_summary.json C2 smsp__inst_executed x 32 / particles"}

    line = {"metric": METRIC, "value": value, "unit": "particle-steps/s", "n_gpus": world, "steps": K,
            "warmup": Wm, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f32", "data": DATA, "config": _config(world), "estimates_per_s": steps_per_s,
            "roofline": roofline, "roofline_issue": roofline_issue,
            "e2e": {"value": e2e_value, "unit": "particle-steps/s", "estimates_per_s": 1e3 / e2e_ms,
                    "ms_per_step": e2e_ms, "h2d_bytes_per_step": 4 * (NJ + 2 + NJ),
                    "d2h_bytes_per_step": 4 * (4 + D)},
            "clocks": clocks, "gpu_launches": K * (1 if (world == 1 or transport["p2p"]) else 2), **extras}
    if shared:
        line["config"]["shared_gpus"] = "functional check: ranks share GPUs (gloo host plumbing); not a timing"
    if world > 1:
        line["config"]["transport"] = ("nvlink peer stores + device rendezvous in the step kernel" if transport["p2p"]
                                       else "nccl send/recv halos + all-gather of records")
    if rank == 0 and world == 1:
        rate, nsteps, particles, times = _oracle_rate(a.cpu_seconds)
        line["cpu_baseline"] = {"value": rate, "unit": "particle-steps/s", "cores": 1, "kind": "oracle",
                                "sample": f"oracle (plain C, 1 thread) on 256 of the 4096 sub-filters x 256 of C2 "
                                          f"({particles} particles), {nsteps} steps"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    args = _args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)
