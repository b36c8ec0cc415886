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
same metric through the C ABI with host inputs and a device->host estimate
read every step, timed on the HOST clock (perf_counter around pf_step +
pf_estimate, the stream idle before each call).  The same run also times,
device-side, the BASELINE configs C5 (16M particles of the medium arm per GPU,
ring t = 1, RWS: weak scaling) and C4 (16M particles of the high-DOF arm in
total, d = 32, Vose: strong scaling), each with its own HBM roofline; with
N > 1 the NCCL transport is timed next to the in-kernel peer transport.
``value`` stays C2 per GPU at every N (one per-GPU workload for the driver's
scaling efficiency); the C4 / C5 curves are the ``c4_strong`` / ``c5_weak``
blocks of the per-N lines.  ``cpu_baseline`` is the oracle on every host core
(one process per core on disjoint sub-filter slices), the single-core number
next to it.  ``--impl reference`` times the same multi-process oracle (the
only other place bench.py runs oracle/) on a bounded sample.
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


def _oracle_rate(seconds: float, steps_cap: int | None = None, n_sample: int = 256, seed: int = 1,
                 warmup: int = 0):
    """Particle-steps/s of the CPU oracle (single thread) on a bounded sample
    of the C2 workload: n_sample sub-filters of 256 particles (its own ring)."""
    from oracle import orc
    from paper_conf_ipps_chitchianasks13_b200 import workload as W
    T = 400
    tr = W.make_trajectory(NJ, T, 0)
    f = orc.Filter(orc.Config(m=M_SUB, n_filters=n_sample, t=T_EX, topo="ring", resampler="rws", seed=seed),
                   orc.Model(n_joints=NJ), tr["mu0"], tr["sigma0"])
    for k in range(1, warmup + 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
        f.estimate()
    times = []
    t_all = time.perf_counter()
    k = warmup + 1
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


def _oracle_worker(job):
    """One host core: the oracle on its own slice of C2 sub-filters."""
    seconds, steps_cap, n_sample, seed, warmup = job
    rate, nsteps, particles, times = _oracle_rate(seconds, steps_cap, n_sample, seed, warmup)
    return rate, nsteps, particles, sum(times)


def _host_cpu() -> dict:
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cpu_model": model, "logical_cpus": os.cpu_count(),
            "usable_cpus": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()}


def _oracle_multicore(seconds: float, steps_cap: int | None = None, n_sample: int = 64, warmup: int = 1):
    """The oracle on every usable host core at once: P processes, each on its
    own slice of n_sample C2 sub-filters (disjoint seeds), started together.
    Aggregate particle-steps/s = sum over processes (they run concurrently)."""
    import multiprocessing as mp
    P = _host_cpu()["usable_cpus"] or 1
    jobs = [(seconds, steps_cap, n_sample, 1000 + i, warmup) for i in range(P)]
    t0 = time.perf_counter()
    with mp.get_context("spawn").Pool(P) as pool:
        res = pool.map(_oracle_worker, jobs)
    wall = time.perf_counter() - t0
    total = sum(r[1] * r[2] for r in res)                 # particle-steps done by all processes
    busy = max(r[3] for r in res)                         # the slowest process' timed seconds
    return {"value": total / busy, "processes": P, "steps_per_process": min(r[1] for r in res),
            "particles_per_process": res[0][2], "wall_s": wall, "per_process_rate_median": statistics.median(
                r[0] for r in res)}


def run_reference(a) -> None:
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    # every host core: W warm-up steps untimed, then K timed steps, each a
    # bounded sample of C2 (64 sub-filters x 256 per process)
    mc = _oracle_multicore(0, steps_cap=a.steps, n_sample=64, warmup=max(a.warmup, 1))
    rate = mc["value"]
    ms = 1e3 * mc["particles_per_process"] * mc["processes"] / rate
    cpu = _host_cpu()
    sample = (f"oracle (plain C) on {mc['processes']} processes x 64 of the 4096 sub-filters x 256 of C2 "
              f"({mc['particles_per_process']} particles each), {a.steps} timed steps each")
    line = {"metric": METRIC, "value": rate, "unit": "particle-steps/s", "impl": "reference",
            "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": DATA,
            "config": _config(1), "estimates_per_s": rate / PARTICLES_PER_GPU,
            "cpu_baseline": {"value": rate, "unit": "particle-steps/s", "cores": mc["processes"], "kind": "oracle",
                             "sample": sample, **cpu},
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


# BASELINE configs timed next to C2: name -> (n_joints, m,
# sub-filters, resampler, scaling).  C5: 2^24 particles PER GPU (weak);
# C4: 2^24 particles IN TOTAL, split over the ranks (strong).
EXTRA_CONFIGS = {
    "c5_weak": (5, 256, 65536, "rws", "weak"),
    "c4_strong": (28, 256, 65536, "vose", "strong"),
}


def _bytes_per_launch(d: int, particles: int, n_sub: int, t: int = T_EX, deg: int = 2) -> int:
    """Algorithmic HBM bytes of one step launch: read + write the
    d + 1 floats of every particle, write the best-t mailbox row of every
    sub-filter, read deg * t mailbox entries per sub-filter."""
    return particles * 8 * (d + 1) + n_sub * t * (d + 2) * 4 * (1 + deg)


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
            # one collective so the communicator exists, then say how many ranks it spans
            chk = torch.ones(1, device=torch.device("cuda", local))
            dist.all_reduce(chk)
            if rank == 0:
                print(f"[bench] NCCL communicator: nranks={dist.get_world_size()} "
                      f"all_reduce(1)={int(chk.item())} backend={dist.get_backend()}", file=sys.stderr, flush=True)
    dev = torch.device("cuda", local)
    K, Wm = a.steps, max(a.warmup, 3)
    T = Wm + K + 8
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = peaks.get("hbm_gbs", 6650.0)
    peak_source = "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"
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
    trajs = {}

    def traj(nj):
        if nj not in trajs:
            tr = W.make_trajectory(nj, T, 0)
            trajs[nj] = (tr, torch.tensor(tr["Z"][1:], device=dev), torch.tensor(tr["U"][:-1], device=dev))
        return trajs[nj]

    transport = {"p2p": False}   # multi-rank: halo + estimate inside the kernel (peer transport) or NCCL

    # ---- device-resident inputs: CUDA events around every step ------------
    def device_run(nj, m, n_sub, resampler, flush_l2, steps, transport_name=None):
        tr, zs, us = traj(nj)
        pf = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=n_sub, t=T_EX,
                              topo="ring", seed=2013, rank=rank, world=world, resampler=resampler,
                              device_inputs=True)
        df = Dd.DistributedFilter(pf, transport=transport_name)
        if transport_name is None:
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
        pf.close()
        del df, pf
        return ms / steps

    ms_step = device_run(NJ, M_SUB, N_SUB * world, "rws", True, K)
    steps_per_s = 1e3 / ms_step
    value = steps_per_s * PARTICLES_PER_GPU * world

    extras = {}
    if not a.no_extras:
        ms_v = device_run(NJ, M_SUB, N_SUB * world, "vose", True, K)
        ms_w = device_run(NJ, M_SUB, N_SUB * world, "rws", False, K)
        # batched mode (SURVEY §8(d) metric (1)): K steps of device-resident z/u in ONE pf_step_batch
        # call, every step's estimate record written on the device, one synchronisation
        tr2, zs2, us2 = traj(NJ)
        if world == 1:
            pfb = F.ParticleFilter(tr2["mu0"], tr2["sigma0"], F.ArmModel(n_joints=NJ), m=M_SUB, n_filters=N_SUB,
                                   t=T_EX, topo="ring", seed=2013, resampler="rws", device_inputs=True)
            est = torch.zeros(K, 4 + D, device=dev)
            pfb.step_batch(zs2[:Wm], us2[:Wm])
            torch.cuda.synchronize()
            eb0, eb1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            eb0.record(pfb.stream)
            pfb.step_batch(zs2[Wm:Wm + K], us2[Wm:Wm + K], est)
            eb1.record(pfb.stream)
            torch.cuda.synchronize()
            ms_b = eb0.elapsed_time(eb1) / K
            pfb.close()
        extras = {"vose": {"estimates_per_s": 1e3 / ms_v, "ms_per_step": ms_v,
                           "particle_steps_per_s": 1e3 / ms_v * PARTICLES_PER_GPU * world},
                  "l2_resident": {"estimates_per_s": 1e3 / ms_w, "ms_per_step": ms_w,
                                  "note": "back-to-back steps, particle set (84 MB) left in the 126 MB L2"}}
        if world == 1:
            extras["batched"] = {"estimates_per_s": 1e3 / ms_b, "ms_per_step": ms_b,
                                 "note": f"pf_step_batch: {K} steps of device-resident inputs in one call, estimate "
                                         "records on the device, one synchronisation (no flush: the set stays in L2)"}
        # BASELINE configs C5 (weak) and C4 (strong), device-timed, L2 flushed
        # (their particle sets, 640 MB / 2.2 GB, exceed the L2 anyway)
        for name, (nj, m, n_sub, res, scaling) in EXTRA_CONFIGS.items():
            n_total = n_sub * world if scaling == "weak" else n_sub
            ms_x = device_run(nj, m, n_total, res, True, K)
            parts_total = n_total * m
            d = nj + 4
            bl = _bytes_per_launch(d, parts_total // world, n_total // world)
            ach = bl / (ms_x * 1e-3) / 1e9
            extras[name] = {
                "workload": (f"{'C5' if name.startswith('c5') else 'C4'}: arm n_joints {nj} (d {d}), "
                             f"{n_total} sub-filters x {m} = {parts_total} particles in total, ring t {T_EX}, {res}"),
                "scaling": scaling, "particles_total": parts_total, "particles_per_gpu": parts_total // world,
                "ms_per_step": ms_x, "particle_steps_per_s": parts_total * 1e3 / ms_x, "estimates_per_s": 1e3 / ms_x,
                "roofline": {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                             "bytes_per_launch_per_gpu": bl, "peak_source": peak_source}}
        if world > 1 and not shared:
            # the NCCL transport (halo send/recv + record all-gather around the step) next to the peer one
            try:
                ms_n = device_run(NJ, M_SUB, N_SUB * world, "rws", True, K, transport_name="nccl")
                extras["nccl_transport"] = {"ms_per_step": ms_n, "particle_steps_per_s": 1e3 / ms_n *
                                            PARTICLES_PER_GPU * world,
                                            "note": "PF_TRANSPORT=nccl: torch.distributed NCCL halos + all-gather "
                                                    "of the per-rank records, same C2 workload"}
            except Exception as exc:   # reported, not fatal: the peer-transport line above stands
                extras["nccl_transport"] = {"error": f"{type(exc).__name__}: {exc}"[:300]}

    # ---- end to end through the C ABI with host buffers, HOST clock --------
    tr, _, _ = traj(NJ)
    pf = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=NJ), m=M_SUB, n_filters=N_SUB * world,
                          t=T_EX, topo="ring", seed=2013, rank=rank, world=world, resampler="rws")
    df = Dd.DistributedFilter(pf)
    Zh = np.ascontiguousarray(tr["Z"][1:], np.float32)
    Uh = np.ascontiguousarray(tr["U"][:-1], np.float32)
    for k in range(Wm):
        df.step(Zh[k], Uh[k])
        df.estimate()
    barrier()
    host_s = []
    sampler.active = True
    for i in range(K):
        flush.zero_()
        torch.cuda.synchronize()               # the stream is idle when the user's call starts
        t0 = time.perf_counter()
        df.step(Zh[Wm + i], Uh[Wm + i])        # H2D of z_k, u_{k-1} (inside the launch) + the step
        df.estimate()                          # D2H of the estimate record (mapped host poll / copy + sync)
        host_s.append(time.perf_counter() - t0)
    sampler.active = False
    sampler.__exit__()
    clocks = sampler.summary()
    barrier()
    e2e_ms = max_over_ranks(1e3 * sum(host_s) / K)
    pf.close()
    e2e_value = 1e3 / e2e_ms * PARTICLES_PER_GPU * world

    # ---- roofline of the step kernel (C2) ------------------------------------
    bytes_launch = _bytes_per_launch(D, PARTICLES_PER_GPU, N_SUB)
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
                "peak_source": peak_source, "note": "issue-bound: see roofline_issue and DESIGN.md §6"}
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
                    "d2h_bytes_per_step": 4 * (4 + D), "clock": "host perf_counter around pf_step + pf_estimate, "
                                                           "stream idle before each call"},
            "clocks": clocks, "gpu_launches": K * (1 if (world == 1 or transport["p2p"]) else 2), **extras}
    if shared:
        line["config"]["shared_gpus"] = "functional check: ranks share GPUs (gloo host plumbing); not a timing"
    if world > 1:
        line["config"]["transport"] = ("nvlink peer stores + device rendezvous in the step kernel" if transport["p2p"]
                                       else "nccl send/recv halos + all-gather of records")
    if rank == 0 and world == 1:
        mc = _oracle_multicore(a.cpu_seconds, n_sample=64)
        rate1, nsteps1, particles1, _ = _oracle_rate(min(a.cpu_seconds, 5.0), n_sample=64)
        line["cpu_baseline"] = {
            "value": mc["value"], "unit": "particle-steps/s", "cores": mc["processes"], "kind": "oracle",
            "sample": (f"oracle (plain C) on all {mc['processes']} usable host cores at once: one process per core, "
                       f"each on its own 64 sub-filters x 256 of C2 ({mc['particles_per_process']} particles), "
                       f">= {mc['steps_per_process']} steps each in {a.cpu_seconds:g} s"),
            "single_core": {"value": rate1, "steps": nsteps1, "particles": particles1},
            **_host_cpu()}
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
