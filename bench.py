#!/usr/bin/env python
"""Benchmark: batched SS-HOPM (solve + dedup [+ NCCL gather]) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

A step is one pass of the whole hot path over one batch: sshopm_solve over
N tensors x S starts, then sshopm_dedup (and, for world size > 1, one NCCL
gather of the fixed-size dedup records to rank 0).  Inputs are resident in
HBM before timing starts; L2 is flushed between timed steps (a 512 MiB write
outside the timed events).  Each rank owns a contiguous tensor range of size
config N (weak scaling); time = max over ranks of the summed per-step CUDA
event durations.  Rank 0 prints ONE JSON line.

value = paper-style GFLOP/s = F_paper(m, n) * sum(iters) / time (reading R12,
SURVEY.md 8(d); lambda_0 excluded).  voxel-solves/s is reported beside it.
roofline: the solve kernel against the FP32 ALU peak
148 SM x 128 lanes x 2 flop x f_max, counting the library's
algorithmic FP32 flops per update (sshopm_flops_per_iter "executed").
"""
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

import synthetic as syn  # noqa: E402

METRIC = "SS-HOPM Gflop/s & voxel-solves/s (m=4,n=3,128 starts) vs FP32 peak"
LAM_TOL, ANG_TOL, KMAX = 1e-2, 0.05, 4


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=sorted(syn.CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--voxels", type=int, default=0, help="override tensors per rank")
    ap.add_argument("--refill", type=int, default=0)
    ap.add_argument("--schedule", type=int, default=0, help="0 library default, 1 item-per-lane, 2 tensor-per-lane")
    ap.add_argument("--unfused", action="store_true", default=True,
                    help="step = sshopm_solve + sshopm_dedup as separate calls (default; the solve is timed alone)")
    ap.add_argument("--solve-dedup", dest="unfused", action="store_false", help="step = one sshopm_solve_dedup call")
    ap.add_argument("--fused", action="store_true", help="sshopm_solve_dedup with in-kernel clustering (opt-in)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-voxels", type=int, default=0)
    ap.add_argument("--e2e-chunk", type=int, default=0, help="tensors per run_host chunk (0: auto)")
    ap.add_argument("--e2e-rep", action="store_true",
                    help="e2e also returns each cluster's representative start (default: the SURVEY 8(e) record "
                         "count | K x (lambda, x, mult), 84 B per tensor for (4,3), K = 4)")
    ap.add_argument("--gather-chunks", type=int, default=0,
                    help="N > 1: solve+dedup the rank's range in C chunks and gather chunk i on a side stream "
                         "while chunk i+1 solves (0: 4 when N > 1, else 1)")
    ap.add_argument("--gather", default="nccl", choices=["nccl", "p2p"],
                    help="N > 1: A9 as NCCL gathers per chunk (default), or p2p: the dedup kernel stores the records "
                         "straight into rank 0's buffer over NVLink (IPC-mapped peer memory, no collective)")
    ap.add_argument("--graph", action="store_true",
                    help="N = 1: capture one step (pack, solve, dedup launches) in a CUDA graph and replay it "
                         "(launch-bound small volumes); the solve is then timed together with the step")
    ap.add_argument("--dump-records", default="", help="rank 0: save the gathered dedup records (.npz) after the run")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process group backend for N > 1 (gloo: exercise the multi-rank path on one GPU)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks --
class ClockSampler:
    """NVML SM-clock / throttle-reason sampler running during the timed region."""
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index, period=0.01):
        self.samples, self.reasons, self.ok = [], set(), False
        self.period = period
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None
        self._stop = threading.Event()

    def _sample(self):
        nv = self.nv
        try:
            self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
            r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h) if hasattr(nv, "nvmlDeviceGetCurrentClocksEventReasons") \
                else nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
            for bit, name in self.REASONS.items():
                if r & bit and name not in ("gpu_idle",):
                    self.reasons.add(name)
        except Exception:
            pass

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h) if hasattr(nv, "nvmlDeviceGetCurrentClocksEventReasons") \
                    else nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name not in ("gpu_idle",):
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def sample_now(self):
        """Explicit sample from the timing loop (the GPU is busy while the host enqueues ahead)."""
        if self.ok:
            self._sample()

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def peaks():
    p = {}
    f = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(f):
        with open(f) as fh:
            p = json.load(fh)
    return p


# --------------------------------------------------------------- CPU oracle --
def _oracle_chunk(args):
    cfg, first, count, seed = args
    from oracle import sshopm as O
    ent = syn.gen_voxels(cfg["m"], cfg["n"], first, count, seed)
    st = syn.gen_starts(cfg["S"], cfg["n"], seed)
    lam, x, it, cv = O.sshopm(ent, st, cfg["m"], cfg["n"], cfg["alpha"], cfg["tol"], cfg["maxit"])
    return int(it.sum()), count


def cpu_oracle(cfg, n_voxels, seed=0, first=0):
    """Time the FP64 oracle as it stands on the host cores (process pool, one process per core)."""
    import multiprocessing as mp
    from oracle.sshopm import paper_flops_per_iter
    cores = len(os.sched_getaffinity(0))
    chunk = 64 if cfg["m"] <= 4 and cfg["n"] <= 3 else 16
    tasks = [(cfg, first + v, min(chunk, n_voxels - v), seed) for v in range(0, n_voxels, chunk)]
    ctx = mp.get_context("fork")
    t0 = time.perf_counter()
    with ctx.Pool(cores) as pool:
        res = pool.map(_oracle_chunk, tasks, chunksize=1)
    dt = time.perf_counter() - t0
    iters = sum(r[0] for r in res)
    F = paper_flops_per_iter(cfg["m"], cfg["n"])
    return {"gflops": F * iters / dt / 1e9, "voxel_solves_per_s": n_voxels / dt, "seconds": dt, "cores": cores,
            "iters": iters, "voxels": n_voxels}


def reference_arm(a, cfg, rank, world):
    """--impl reference: the oracle (FP64 CPU) timed on host cores, rank 0 only."""
    if rank != 0:
        return
    nvox = a.cpu_voxels or (16384 if (cfg["m"], cfg["n"]) == (4, 3) else 1024)
    for _ in range(a.warmup):
        cpu_oracle(cfg, min(nvox, 256))
    tot_t, tot_it, tot_v = 0.0, 0, 0
    cores = None
    for s in range(a.steps):
        r = cpu_oracle(cfg, nvox, seed=0, first=s * nvox)
        tot_t += r["seconds"]
        tot_it += r["iters"]
        tot_v += r["voxels"]
        cores = r["cores"]
    from oracle.sshopm import paper_flops_per_iter
    F = paper_flops_per_iter(cfg["m"], cfg["n"])
    val = F * tot_it / tot_t / 1e9
    sample = f"{nvox} tensors x {cfg['S']} starts per step (of {cfg['N']}), FP64 full-tensor numpy oracle, process pool"
    line = {"metric": METRIC, "value": val, "unit": "GFLOP/s", "impl": "reference", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * tot_t / a.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": a.config, "m": cfg["m"], "n": cfg["n"], "tensors": cfg["N"], "starts": cfg["S"],
                       "alpha": cfg["alpha"], "tol": cfg["tol"], "maxit": cfg["maxit"]},
            "voxel_solves_per_s": tot_v / tot_t,
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- launcher --
def free_port():
    import socket
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def launch_command(argv, n, port):
    """torchrun command line that re-runs this script with the same arguments on n local ranks."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
            "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + list(argv)


def self_launch(a, argv):
    """`python bench.py --gpus N` (N > 1) outside torchrun: start the N ranks ourselves, one process per
    GPU, and return their exit status.  Under torchrun (WORLD_SIZE set) the world size must equal --gpus."""
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is not None:
        if int(world_env) != a.gpus and "--gpus" in " ".join(argv):
            raise SystemExit(f"bench.py: WORLD_SIZE={world_env} but --gpus {a.gpus}")
        return None
    if a.gpus <= 1:
        return None
    env = dict(os.environ)
    # NCCL's communicator-init log (ranks, NVLS / NVLink topology) goes to files, not to the JSON stdout
    if a.backend == "nccl" and "NCCL_DEBUG" not in env:
        os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
        env.update(NCCL_DEBUG="INFO", NCCL_DEBUG_SUBSYS="INIT",
                   NCCL_DEBUG_FILE=os.path.join(ROOT, "gpurun_out", "nccl_init.%h.%p.log"))
    import subprocess
    return subprocess.run(launch_command(argv, a.gpus, free_port()), env=env).returncode


# ---------------------------------------------------------------- our arm --
def main():
    a = parse()
    rc = self_launch(a, sys.argv[1:])
    if rc is not None:
        return rc
    cfg = dict(syn.CONFIGS[a.config])
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if a.voxels:
        cfg["N"] = a.voxels
    if a.impl == "reference":
        return reference_arm(a, cfg, rank, world)

    import torch
    import torch.distributed as dist
    import paper_conf_ipps_ballardkp11_b200 as sh
    from paper_conf_ipps_ballardkp11_b200 import sharding as SH

    local = local % torch.cuda.device_count()           # gloo test runs may share one GPU
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if a.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    m, n, S, Nloc = cfg["m"], cfg["n"], cfg["S"], cfg["N"]
    strong = bool(cfg.get("total")) and not a.voxels     # C5: fixed whole volume split over the ranks
    if strong:
        assert Nloc % world == 0, "strong-scaling config: tensors must divide evenly over the ranks"
        Nloc //= world
    solver = sh.Solver(m, n)
    U = solver.U

    # inputs: this rank's tensor range (counter-based generator -> shard invariant), resident in HBM
    first, count = SH.shard_range(Nloc * world, rank, world)
    assert count == Nloc
    ent_h = syn.gen_voxels(m, n, first, Nloc, seed=0)
    st_h = syn.gen_starts(S, n, seed=0)
    ent = torch.from_numpy(ent_h).to(dev)
    st = torch.from_numpy(st_h).to(dev)
    lam = torch.empty((Nloc, S), dtype=torch.float32, device=dev)
    xo = torch.empty((Nloc, S, n), dtype=torch.float32, device=dev)
    it = torch.empty((Nloc, S), dtype=torch.int32, device=dev)
    cv = torch.empty((Nloc, S), dtype=torch.uint8, device=dev)
    # dedup records: one int32 block per chunk so one collective moves a chunk (sharding.py); with
    # N > 1 chunk c's gather runs on a side stream while chunk c+1 solves (SURVEY.md 8(e) overlap)
    n_chunks = a.gather_chunks or (4 if world > 1 else 1)
    bounds = SH.chunk_bounds(Nloc, n_chunks)
    n_chunks = len(bounds)
    peer = None
    if world > 1 and a.gather == "p2p":
        peer = SH.PeerRecords(Nloc, n_chunks, KMAX, n, rank, world, dev)
        blocks = peer.blocks                              # this rank's slice of rank 0's buffer
    else:
        rec = torch.empty(SH.chunked_record_words(Nloc, n_chunks, KMAX, n)[0], dtype=torch.int32, device=dev)
        blocks = SH.chunked_record_views(rec, Nloc, n_chunks, KMAX, n)
    titers = torch.zeros(1, dtype=torch.int64, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    side = torch.cuda.Stream(device=dev)
    done = [torch.cuda.Event() for _ in range(n_chunks)]
    gathered = [None] * n_chunks

    def run_chunk(c, count_iters=False, ev=None):
        """One pass of the hot path over chunk c: solve (A0-A7) + dedup (A8).  ev = (start, mid) events
        recorded around the solve launches (two-pass forms) so the solve kernel is timed on its own."""
        ti = titers if count_iters else None
        v0, v1 = bounds[c]
        views = blocks[c][1]
        o = (lam[v0:v1], xo[v0:v1], it[v0:v1], cv[v0:v1])
        if ev is not None:
            ev[0].record(stream)
        if a.unfused:
            solver.solve(ent[v0:v1], st, cfg["alpha"], cfg["tol"], cfg["maxit"], out=o,
                         refill_threshold=a.refill, total_iters=ti, schedule=a.schedule)
            if ev is not None:
                ev[1].record(stream)
            solver.dedup(*o[:2], o[3], LAM_TOL, ANG_TOL, KMAX, out=tuple(views))
        else:
            solver.solve_dedup(ent[v0:v1], st, cfg["alpha"], cfg["tol"], cfg["maxit"], LAM_TOL, ANG_TOL, KMAX,
                               out=o, dedup_out=tuple(views), refill_threshold=a.refill,
                               total_iters=ti, schedule=a.schedule, fused=a.fused)
            if ev is not None:
                ev[1].record(stream)
        if world > 1 and peer is None:
            gather(c)

    def gather(c):
        block = blocks[c][0]
        if a.backend == "nccl":                           # A9: NCCL gather of chunk c on the side stream
            done[c].record(stream)
            with torch.cuda.stream(side):
                side.wait_event(done[c])
                gathered[c] = SH.gather_records(block, rank, world)
        else:                                             # gloo: stage through host memory (no overlap)
            gathered[c] = SH.gather_records(block.cpu(), rank, world)

    def run_path(count_iters=False, evs=None):
        for c in range(n_chunks):
            run_chunk(c, count_iters, None if evs is None else evs[c])
        if world > 1 and peer is None:
            stream.wait_stream(side)                      # the step ends when the last gather has landed

    def step(count_iters=False):
        if count_iters:
            titers.zero_()
        run_path(count_iters)

    for _ in range(max(a.warmup, 3)):
        step()
    step(count_iters=True)
    torch.cuda.synchronize()
    iters_local = int(titers.item())

    graph = None
    if a.graph:
        assert world == 1, "--graph is for N = 1"
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream(device=dev)
        cap.wait_stream(stream)
        with torch.cuda.stream(cap):
            run_path()                                    # warm the capture stream (workspaces, caches)
            cap.synchronize()
            lc0 = solver.launch_count()
            with torch.cuda.graph(graph, stream=cap):
                run_path()
            launches_per_replay = solver.launch_count() - lc0
        stream.wait_stream(cap)
        torch.cuda.synchronize()

    def tev():
        return torch.cuda.Event(enable_timing=True)
    ev = [(tev(), tev()) for _ in range(a.steps)]
    cev = [[(tev(), tev()) for _ in range(n_chunks)] for _ in range(a.steps)]   # per-chunk solve windows
    l0 = solver.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for i in range(a.steps):
            if i % 4 == 2:
                clk.sample_now()                          # host-side NVML query: outside the event window
            flush.zero_()
            e0, e2 = ev[i]
            e0.record(stream)
            if graph is not None:
                graph.replay()
                cev[i][0][0].record(stream)               # no solve-only window inside a graph
                cev[i][0][1].record(stream)
            else:
                run_path(evs=cev[i])
            e2.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches = solver.launch_count() - l0
    if graph is not None:
        launches = launches_per_replay * a.steps          # kernels inside each replayed graph
    t_step = [e0.elapsed_time(e2) for e0, e2 in ev]
    # pack + solve kernels of every chunk (with --solve-dedup: the whole call)
    t_solve = [sum(s0.elapsed_time(s1) for s0, s1 in cs) for cs in cev]
    if graph is not None:
        t_solve = t_step                                  # roofline over the whole replayed step (conservative)
    tot_ms = float(sum(t_step))
    cdev = dev if a.backend == "nccl" else torch.device("cpu")
    stats = torch.tensor([tot_ms, float(iters_local), float(sum(t_solve))], dtype=torch.float64, device=cdev)
    if world > 1:
        tmax = stats[[0, 2]].clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        itsum = stats[1:2].clone()
        dist.all_reduce(itsum, op=dist.ReduceOp.SUM)
        tot_ms, solve_ms, iters_all = float(tmax[0]), float(tmax[1]), float(itsum[0])
    else:
        solve_ms, iters_all = float(stats[2]), float(stats[1])

    if a.dump_records and world > 1 and peer is not None:
        torch.cuda.synchronize()
        dist.barrier()                                    # every rank's dedup stores have landed in rank 0's buffer
    if a.dump_records and rank == 0:
        if world > 1 and peer is not None:
            merged = peer.merged()
        elif world > 1:
            merged = SH.merge_chunked(gathered, Nloc, n_chunks, KMAX, n)
        else:
            merged = SH.merge_chunked([[blk] for blk, _ in blocks], Nloc, n_chunks, KMAX, n)
        np.savez(a.dump_records, **dict(zip(("count", "lam", "x", "mult", "rep"), merged)))

    # end to end through the C ABI on host buffers (pinned), per step
    e2e = None
    if not a.no_e2e:
        ent_p = torch.from_numpy(ent_h).pin_memory()
        st_p = torch.from_numpy(st_h).pin_memory()
        outs = {"count": torch.empty(Nloc, dtype=torch.int32).pin_memory(),
                "lambda": torch.empty((Nloc, KMAX), dtype=torch.float32).pin_memory(),
                "x": torch.empty((Nloc, KMAX, n), dtype=torch.float32).pin_memory(),
                "mult": torch.empty((Nloc, KMAX), dtype=torch.int32).pin_memory()}
        if a.e2e_rep:                                     # representative start per cluster (diagnostic)
            outs["rep"] = torch.empty((Nloc, KMAX), dtype=torch.int32).pin_memory()
        chunk = a.e2e_chunk or min(Nloc, min(262144, max(65536, Nloc // 8)))   # the library default (host_pipeline.cu)
        solver.run_host(ent_p, st_p, cfg["alpha"], cfg["tol"], cfg["maxit"], LAM_TOL, ANG_TOL, KMAX,
                        chunk_tensors=chunk, out=outs)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(a.steps):
            solver.run_host(ent_p, st_p, cfg["alpha"], cfg["tol"], cfg["maxit"], LAM_TOL, ANG_TOL, KMAX,
                            chunk_tensors=chunk, out=outs)
        e2e_s = time.perf_counter() - t0
        e2e_t = torch.tensor([e2e_s], dtype=torch.float64, device=dev if a.backend == "nccl" else "cpu")
        if world > 1:
            dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        e2e_s = float(e2e_t[0])
        h2d = ent_h.nbytes + st_h.nbytes
        d2h = sum(int(v.numel() * v.element_size()) for k, v in outs.items() if k != "total_iters")
        F = solver.paper_flops_per_iter
        e2e = {"value": F * iters_all * a.steps / e2e_s / 1e9, "unit": "GFLOP/s", "h2d_bytes_per_step": h2d * world,
               "d2h_bytes_per_step": d2h * world, "ms_per_step": 1e3 * e2e_s / a.steps,
               "voxel_solves_per_s": Nloc * world * a.steps / e2e_s, "chunk_tensors": chunk}

    if rank != 0:
        if world > 1:
            if peer is not None:
                dist.barrier()                            # rank 0 unmaps last
                peer.close()
            dist.destroy_process_group()
        return

    F = solver.paper_flops_per_iter
    Fx = solver.exec_flops_per_iter - (2 * n if cfg["alpha"] == 0 else 0)   # alpha = 0: no shift flops
    T = tot_ms / 1e3
    value = F * iters_all * a.steps / T / 1e9
    vps = Nloc * world * a.steps / T
    pk = peaks()
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    fmax = pk.get("sm_max_mhz") or clk.max_mhz or 1965.0
    peak_tflops = sms * 128 * 2 * fmax * 1e6 / 1e12
    # algorithmic flops of one solve: every (tensor, start) lane evaluates lambda_0 = x_0 . A x_0^{m-1}
    # (reading R1) and then, per update k = 1..iters, one normalisation (+ shift) and one evaluation:
    # Fx per update + Fe for lambda_0; paper-style `value` keeps lambda_0 excluded (R12)
    Fu = (2 * n - 1) + n + (2 * n if cfg["alpha"] != 0 else 0)          # ||xhat||^2, scale, shift
    Fe = Fx - Fu                                                          # monomials + 2*T1 + lambda
    alg_flops = Fx * iters_local + Fe * Nloc * S
    achieved = alg_flops * a.steps / (solve_ms / 1e3) / 1e12             # rank-local solve kernel
    traffic = fma_pct = exec_gflop = None
    tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tf):
        with open(tf) as fh:
            prof = json.load(fh)
        traffic = prof.get(a.config)
        fma_pct = prof.get(a.config + "_fma_pipe_active_pct")
        exec_gflop = prof.get(a.config + "_executed_fp32_gflop")
    # SURVEY 8(d) metrics 6-7 from the last step's outputs (outside the timed region): converged
    # fraction, dedup cluster histogram, executed-flop fraction (ncu count / this run's solve time),
    # voxel-solves/s against the peak-equivalent rate peak / (F_paper x mean iters x S)
    conv_frac = float(cv.float().mean().item())
    counts = torch.cat([blk[1][0] for blk in blocks]).to(torch.int64)
    hist = torch.bincount(counts.clamp(max=KMAX + 1), minlength=KMAX + 2).cpu().tolist()
    mean_it = iters_all / (Nloc * world * S)
    cpu = None
    if world == 1 and not a.no_cpu:
        nv = a.cpu_voxels or (16384 if (m, n) == (4, 3) else 512)
        r = cpu_oracle(cfg, min(nv, Nloc))
        cpu = {"value": r["gflops"], "unit": "GFLOP/s", "cores": r["cores"], "kind": "oracle",
               "sample": f"first {r['voxels']} of {Nloc} tensors x {S} starts (same workload), FP64 full-tensor "
                         f"numpy oracle, {r['cores']} processes, {r['seconds']:.1f} s",
               "voxel_solves_per_s": r["voxel_solves_per_s"]}
    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": tot_ms / a.steps, "higher_is_better": True, "scaling": "strong" if strong else "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": a.config, "m": m, "n": n, "tensors_per_gpu": Nloc, "tensors_total": Nloc * world,
                   "starts": S, "alpha": cfg["alpha"], "tol": cfg["tol"], "maxit": cfg["maxit"],
                   "dedup": {"lam_tol": LAM_TOL, "ang_tol": ANG_TOL, "kmax": KMAX},
                   "flop_count": "paper-style F_paper(m,n) x sum(iters), reading R12",
                   "l2": "flushed between timed steps (512 MiB write outside the events)",
                   "cuda_graph": bool(graph is not None),
                   "parallelism": f"tensor-range shards x{world}" +
                                  ((" + dedup records stored by the dedup kernel into rank 0's memory over "
                                    "peer mappings (p2p, no collective)") if world > 1 and peer is not None else
                                   (f" + {a.backend.upper()} gather of dedup records in {n_chunks} chunks "
                                    f"(chunk i gathered while chunk i+1 solves)" if world > 1 else ""))},
        "voxel_solves_per_s": vps,
        "start_solves_per_s": vps * S,
        "mean_iters": mean_it,
        "converged_frac": conv_frac,
        "dedup_clusters_hist": {str(k) if k <= KMAX else f">{KMAX}": v for k, v in enumerate(hist)},
        "voxel_solves_frac_of_peak_equiv": vps / (peak_tflops * 1e12 / (F * mean_it * S)),
        "value_note": "value and voxel_solves_frac_of_peak_equiv use the paper-style flop count (reading R12: "
                      f"{F} flops per update for ({m},{n}), about 2.8x the FP32 work the kernel executes for (4,3)); "
                      "they are comparable to the paper's 318 GFLOP/s, not a fraction of peak. The fraction of the FP32 "
                      "peak is roofline.frac (algorithmic flops) and roofline.executed_frac_ncu (executed flops).",
        "ms_solve_per_step": solve_ms / a.steps,
        "roofline": {"bound": "alu", "achieved": achieved, "peak": peak_tflops, "unit": "TFLOP/s",
                     "frac": achieved / peak_tflops, "traffic": traffic,
                     "frac_updates_only": Fx * iters_local * a.steps / (solve_ms / 1e3) / 1e12 / peak_tflops,
                     "kernel": f"sshopm_solve_kernel<{m},{n}>",
                     "peak_basis": f"{sms} SM x 128 FP32 lanes x 2 x {fmax:.0f} MHz (sm_max_mhz)",
                     "flops_per_update": Fx, "flops_lambda0_eval": Fe,
                     "flops_per_launch": alg_flops,
                     "fma_pipe_active_pct_ncu": fma_pct,
                     "executed_frac_ncu": (exec_gflop * 1e9 / (solve_ms / a.steps / 1e3) / 1e12 / peak_tflops
                                           if exec_gflop and world == 1 else None),
                     "flops_note": "algorithmic FP32 flops per launch = flops_per_update x sum(iters) + flops_lambda0_eval x N*S "
                                   "(update: monomials + 2*T1 + lambda + shift + norm + scale; lambda_0: monomials + 2*T1 + lambda; DESIGN.md 7); "
                                   "frac_updates_only counts the updates alone (lambda_0 evaluations as free work)"},
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "context": {"paper_gpu": "318 GFLOP/s paper-style (31% of 1030), Tesla C2050, 1024 tensors (P:L5, P:L350)"},
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        if peer is not None:
            dist.barrier()
            peer.close()
        dist.destroy_process_group()


if __name__ == "__main__":
    sys.exit(main() or 0)
