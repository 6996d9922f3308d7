#!/usr/bin/env python3
"""Benchmark: GCUPS of the Smith-Waterman database search on B200 (BASELINE.json metric).

One STEP = the whole hot path (profile build, both regimes, 32-bit recompute, scatter to
caller order, and for N > 1 the NCCL score gather) for the 5 queries of config C2
(lengths 144/375/729/1500/5478, BLOSUM62, gap open 10 / extend 2, threshold 3072) against
a Swiss-Prot-shaped synthetic database of 540,000 sequences (~191M residues) PER GPU.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C2|C1|C3|C4|C5]
  python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N

value   = sum_q m_q * sum_j n_j (all ranks) / max-over-ranks device time of K steps (GCUPS);
e2e     = same metric through the blocking host API (sw_search_batch: queries H2D, scores D2H);
roofline= the fused search kernel (k_search) against the derived ALU-pipe bound
          (tools/int_peaks.cu -> MEASURED_INT_PEAKS.json), clock-normalised;
parity  = rank 0 compares a deterministic sample of the step's scores (global order, after the
          gather) with the CPU oracle; any mismatch exits non-zero;
cpu_baseline = the CPU oracle (oracle/, OpenMP, all host cores) timed on that sample.

Configs: C2 (default) = 540k sequences PER GPU (weak scaling); C4 = C2's 540k-sequence database
split over the N GPUs (strong scaling); C5 = the TrEMBL-scale recipe.
--impl reference times that oracle as the reference arm (the paper ships no code).
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

from workloads import gen  # noqa: E402
from workloads.matrices import MATRICES  # noqa: E402

PAPER_CONTEXT = "PAPER.md: CUDASW++ 17 GCUPS (Tesla C1060, T=3072), >21 GCUPS with the improved kernel (C2050, TAIR)"


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


# ------------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) < 7:
                continue
            try:
                sm.append(float(p[0]))
                mx = float(p[1])
            except ValueError:
                continue
            for n, v in zip(names, p[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# ------------------------------------------------------------------------------- workload
DB_DESC = {"C1": "Swiss-Prot-shaped synthetic DB (parity-small)", "C2": "Swiss-Prot-shaped synthetic DB",
           "C5": "TrEMBL-scale synthetic DB (50M seqs, mean 320), the GPUs' shards of C5_SHARDS",
           "C4": "C2's Swiss-Prot-shaped synthetic DB (540k seqs) split over the GPUs",
           "C3": "long-sequence synthetic DB (all > 3072 residues)"}
SCALING = {"C4": "strong"}   # every other config: weak (a config-sized database per GPU)


def make_workload(name: str, rank: int, world: int, n_override: int | None = None, shard: bool = True):
    """C4: the N ranks split C2's database (strong scaling).  Every other config is weak
    scaling: N ranks search N x (the config's database), one config-sized shard each.
    Returns (queries, this rank's shard (None if not shard), all lengths, matrix, rho, sigma, T,
    seed)."""
    if name == "C4":
        qs = [gen.make_query(L) for L in gen.C2_QUERY_LENGTHS]
        lens = gen.sp_lengths(n_override or 540_000, seed=2)
        seed, mat, T = 2, "BLOSUM62", 3072
    elif name == "C2":
        qs = [gen.make_query(L) for L in gen.C2_QUERY_LENGTHS]
        lens = gen.sp_lengths((n_override or 540_000) * world, seed=2)
        seed, mat, T = 2, "BLOSUM62", 3072
    elif name == "C1":
        qs = [gen.make_query(144)]
        lens = gen.sp_lengths(20_000 * world, seed=1)
        seed, mat, T = 1, "BLOSUM62", 3072
    elif name == "C3":
        qs = [gen.make_query(L) for L in gen.C2_QUERY_LENGTHS]
        lens = gen.long_lengths(4096 * world, seed=3)
        seed, mat, T = 3, "BLOSUM62", 3072
    elif name == "C5":
        # TrEMBL-scale (50M sequences, ~16G residues, BLOSUM45, the 20 benchmark queries): the
        # GPUs of this run search shards 0..N-1 of the database cut into C5_SHARDS round-robin
        # shards (8 = the 8-GPU box; default 64 so one GPU's line takes seconds, not minutes)
        qs = [gen.make_query(L) for L in gen.BENCH_QUERY_LENGTHS]
        full = gen.sp_lengths(50_000_000, seed=5, mu=5.4270)
        n_sh = max(world, int(os.environ.get("C5_SHARDS", "64")))
        order = np.argsort(-full, kind="stable")
        view = np.sort(np.concatenate([order[r::n_sh] for r in range(world)]))
        lens = full[view]
        seed, mat, T = 5, "BLOSUM45", 3072
    else:
        raise SystemExit(f"unknown config {name}")
    db = gen.build_database(lens, seed, qs, sel=gen.shard_indices(lens, rank, world)) if shard else None
    return qs, db, lens, mat, 10, 2, T, seed


def cells_of(qs, total_residues):
    return int(sum(int(q.size) for q in qs)) * int(total_residues)


# ------------------------------------------------------------------------------- cpu oracle
def oracle_sample(qs, lens_all, seed, budget_s: float, cores: int, n_longest: int = 16):
    """Deterministic sample of the GLOBAL database sized for ~budget_s of oracle time on
    `cores`: every k-th sequence plus the n_longest longest (the long regime).  The residues are
    generated from the counter-based recipe (workloads/gen.py), so any rank can build them."""
    per_core = 0.30e9  # cells/s/core of the scalar oracle (SURVEY.md §8(d) measured 0.32-0.36)
    target_cells = budget_s * per_core * cores
    sum_m = sum(int(q.size) for q in qs)
    L = np.asarray(lens_all, dtype=np.int64)
    longest = np.argsort(-L, kind="stable")[:n_longest]
    target_res = max(1, int(target_cells / sum_m) - int(L[longest].sum()))
    stride = max(1, int(L.sum() // target_res))
    idx = np.unique(np.concatenate([np.arange(0, L.shape[0], stride), longest])).astype(np.int64)
    sdb = gen.build_database(L, seed, qs, sel=idx)
    desc = (f"every {stride}-th sequence + the {n_longest} longest of the database "
            f"({idx.size} seqs, {sdb.total_residues} residues) x all {len(qs)} queries")
    return idx, sdb.residues, sdb.offsets, desc


def run_oracle_step(qs, W, rho, sigma, res, off, threads):
    """One oracle pass over the sample: (seconds, [scores per query])."""
    import oracle
    t0 = time.perf_counter()
    out = [oracle.scores(q, W, rho, sigma, res, off, threads=threads) for q in qs]
    return time.perf_counter() - t0, out


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


# ------------------------------------------------------------------------------- reference arm
def bench_reference(args, rank, world):
    if rank != 0:
        return
    qs, _, lens_all, mat, rho, sigma, T, seed = make_workload(args.config, 0, 1, shard=False)
    W = MATRICES[mat]
    cores = cpu_cores()
    budget = max(1.0, 150.0 / max(1, args.steps + args.warmup))
    idx, res, off, desc = oracle_sample(qs, lens_all, seed, budget, cores)
    cells = cells_of(qs, int(off[-1]))
    for _ in range(args.warmup):
        run_oracle_step(qs, W, rho, sigma, res, off, cores)
    times = [run_oracle_step(qs, W, rho, sigma, res, off, cores)[0] for _ in range(args.steps)]
    tot = sum(times)
    gcups = cells * args.steps / tot / 1e9
    line = {
        "impl": "reference", "metric": "GCUPS", "value": round(gcups, 4), "unit": "GCUPS", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * tot / args.steps, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"{args.config} oracle sample", "sample": desc, "queries": [int(q.size) for q in qs],
                   "matrix": mat, "gap_open": rho, "gap_extend": sigma},
        "cpu_baseline": {"value": round(gcups, 4), "unit": "GCUPS", "cores": cores, "cpu_model": cpu_model(),
                         "kind": "oracle", "sample": desc},
        "e2e": {"value": round(gcups, 4), "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------- our arm
def load_int_peaks():
    p = os.path.join(ROOT, "MEASURED_INT_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return None


def bench_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_hainscobr11_b200 as swp
    from paper_conf_ipps_hainscobr11_b200 import build as swbuild

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    # the NCCL path (process group + score gather) runs for N > 1; SW_BENCH_DIST=1 also runs it
    # at N = 1 under torchrun (a one-GPU check of the multi-GPU code path)
    dist_on = world > 1 or os.environ.get("SW_BENCH_DIST") == "1"
    if dist_on:
        # NCCL's own log of communicator set-up (rank count, transports) to stderr, so the
        # stdout JSON line stays alone
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        dist.init_process_group("nccl", device_id=dev)
    if rank == 0:
        swbuild.build()
    if dist_on:
        dist.barrier()
    qs, db, lens_all, mat, rho, sigma, T, seed = make_workload(args.config, rank, world)
    if args.threshold is not None:
        T = -1 if str(args.threshold) == "auto" else int(args.threshold)
    W = MATRICES[mat]
    nq = len(qs)
    from paper_conf_ipps_hainscobr11_b200.dist import ScoreGather, shard_size_bound

    n_total = int(lens_all.shape[0])
    n_local = db.num_seqs
    n_pad = shard_size_bound(n_total, world)
    sw = swp.SmithWaterman(qs[0], W, rho, sigma)
    dist_info = None
    if dist_on:
        gath = ScoreGather(db.global_index, n_total, nq, device=dev)
        # shard padded with empty sequences to the uniform gather size (they score 0)
        sw.load_db(db.residues, ScoreGather.pad_offsets(db.offsets, n_pad))
        out_ptr = gath.send_ptr()
        ranks = [None] * world
        props = torch.cuda.get_device_properties(dev)
        dist.all_gather_object(ranks, {"rank": rank, "device": str(getattr(props, "uuid", local_rank)),
                                       "seqs": n_local, "residues": db.total_residues})
        dist_info = {"backend": dist.get_backend(), "world": dist.get_world_size(), "ranks": ranks,
                     "collective": "gather of int32 score shards to rank 0 (one per step)",
                     "nccl_log": "NCCL_DEBUG=INFO (INIT) on stderr"}
    else:
        gath = None
        sw.load_db(db.residues, db.offsets)
        scores = torch.zeros((nq, n_local), dtype=torch.int32, device=dev)
        out_ptr = scores.data_ptr()
    stream = torch.cuda.current_stream(dev)
    sptr = stream.cuda_stream

    cells_local = cells_of(qs, db.total_residues)
    cells_total = cells_of(qs, int(lens_all.sum()))

    def step(thr=None):
        sw.search_batch_into(qs, out_ptr, T if thr is None else thr, sptr)
        if gath is not None:
            gath.gather()   # NCCL gather of the int32 score shards to rank 0

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if dist_on:
        dist.barrier()
    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    kern_ms = 0.0
    rec_ms = 0.0
    torch.cuda.synchronize(dev)
    if dist_on:
        dist.barrier()
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize(dev)
    ms = ev0.elapsed_time(ev1)
    st = sw.stats()
    clk = clocks.stop()
    # the scores of the last timed step, in global order (rank 0), for the parity check
    if rank == 0:
        step_scores = (gath.to_global() if gath is not None else scores).cpu().numpy()
    # Same step with the library's automatic threshold (SW_AUTO_THRESHOLD),
    # reported beside the configured T (the headline value keeps the config's threshold).
    auto_ms = None
    if T != -1 and not args.no_auto:
        step(-1)
        torch.cuda.synchronize(dev)
        if dist_on:
            dist.barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            step(-1)
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        auto_ms = ev0.elapsed_time(ev1)
        if dist_on:
            t = torch.tensor([auto_ms], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            auto_ms = float(t.item())
    if rank == 0:
        auto_scores = (gath.to_global() if gath is not None else scores).cpu().numpy() if auto_ms else None
    # Dominant-kernel time: one more step with the queries serialised on one stream, so the
    # CUDA events around each fused k_search launch (recorded by the library on the launching
    # stream) time that launch alone; achieved = algorithmic cells / sum of launch durations.
    os.environ["SW_STREAMS"] = "1"
    step()
    torch.cuda.synchronize(dev)
    os.environ.pop("SW_STREAMS", None)
    km = sw.kernel_ms()
    kern_ms, rec_ms = km["search_ms"], km["recompute_ms"]
    if dist_on:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    # end-to-end through the blocking host API (queries H2D, scores D2H), rank-local + max
    # (per-step host wall times, median: one step's time is not skewed by unrelated host load)
    # the scores land in a pinned host buffer reused across steps (the e2e contract's pinned
    # host memory; a fresh pageable array per call spent ~2 ms per step in page faults)
    host_out = torch.empty((len(qs), sw.num_seqs), dtype=torch.int32, pin_memory=True).numpy()
    e2e_times = []
    for _ in range(max(1, args.steps)):
        t0 = time.perf_counter()
        host = sw.search_batch(qs, T, out=host_out)
        if dist_on:
            dist.barrier()
        e2e_times.append(time.perf_counter() - t0)
    e2e_s = float(np.median(e2e_times))
    if dist_on:
        t = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    h2d = int(sum(int(q.size) for q in qs)) + 8 * (nq + 1)
    d2h = int(host.size) * 4

    # streamed database: the same query batch against the
    # HOST-resident shard, chunks sorted/packed/uploaded while the previous chunk is searched
    stream_db = None
    if not args.no_stream:
        chunk = 1 << 28      # ramps 32M, 64M, 128M, ... (profiles/r01_stream_chunk_sweep.jsonl)
        sw.search_stream(db.residues, db.offsets, T, chunk, queries=qs)      # warm: pinned staging
        t0 = time.perf_counter()
        streamed = sw.search_stream(db.residues, db.offsets, T, chunk, queries=qs)
        st_s = time.perf_counter() - t0
        if dist_on:
            t = torch.tensor([st_s], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            st_s = float(t.item())
        stream_db = {"value": round(cells_total / st_s / 1e9, 2), "unit": "GCUPS", "seconds": round(st_s, 4),
                     "chunk_residues": chunk,
                     "h2d_bytes_per_step": int(db.total_residues + 8 * (db.num_seqs + 1)
                                               + sum(int(q.size) for q in qs)),
                     "d2h_bytes_per_step": 4 * nq * db.num_seqs,
                     "api": "sw_search_stream (host DB: sort/pack/upload per chunk, overlapped with the search)"}

    # the host-API outputs must equal the device-timed step's (rank-local shard)
    if gath is None:
        dev_local = step_scores
    else:
        dev_local = gath.send.cpu().numpy()
    local_ok = bool(np.array_equal(host[:, :n_local], dev_local[:, :n_local]))
    if stream_db is not None:
        local_ok = local_ok and bool(np.array_equal(streamed, dev_local[:, :n_local]))
    if dist_on:
        t = torch.tensor([0 if local_ok else 1], dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        local_bad_ranks = int(t.item())
    else:
        local_bad_ranks = 0 if local_ok else 1

    if rank != 0:
        sw.close()
        if dist_on:
            dist.destroy_process_group()
        return
    step_s = ms / 1e3 / args.steps
    gcups = cells_total / step_s / 1e9
    e2e_gcups = cells_total / e2e_s / 1e9

    # roofline of the dominant kernel: the fused k_search launches of the last step
    peaks = load_int_peaks()
    achieved = cells_local / (kern_ms / 1e3) / 1e9 if kern_ms > 0 else None
    roof = {"bound": "alu", "unit": "GCUPS", "achieved": round(achieved, 2) if achieved else None,
            "peak": None, "frac": None, "traffic": None,
            "kernel": f"k_search (fused inter/intra-task); cells of the {nq} launches of one step / their summed "
                      "CUDA-event durations, launches serialised on one stream (SW_STREAMS=1)"}
    if peaks and achieved:
        f_mhz = clk.get("sm_mhz") or peaks.get("sm_mhz_during") or 1965.0
        der = peaks["derived"]
        per_clk = der["cells_per_clk_per_gpu"]
        peak = per_clk * f_mhz * 1e6 / 1e9
        mix = peaks["measured_mix_cells_per_clk_per_gpu"] * f_mhz * 1e6 / 1e9
        conc = cells_local / (step_s * 1e9)   # per-GPU cells over the headline's concurrent step
        roof.update({"peak": round(peak, 1), "frac": round(achieved / peak, 4),
                     "peak_basis": f"derived ALU-pipe bound: {der['alu_pipe_warp_instr_per_clk_per_sm']} warp-instr/clk/SM "
                                   f"(measured, = guide rt_SMSP 2) x 64 cells / {der['alu_ops_per_cell_pair']} ALU ops per "
                                   f"cell pair = {per_clk:.1f} cells/clk/GPU x SM clock {f_mhz:.0f} MHz during the run",
                     "measured_mix_peak": round(mix, 1), "frac_of_measured_mix": round(achieved / mix, 4),
                     "achieved_concurrent": round(conc, 2), "frac_concurrent": round(conc / peak, 4),
                     "concurrent_basis": "headline mode (4 internal query streams): per-GPU cells of the whole step "
                                         "/ the device-timed step (all kernels incl. profile, T-mode, recompute)",
                     "paper_roofline": "SURVEY.md §8(d): measured VIADDMNMX.S16x2 rate x 2 / 6 per cell = "
                                       f"{round(1.998 * 32 * 148 * f_mhz * 1e6 / 3 / 1e9, 1)} GCUPS; frac "
                                       f"{round(achieved / (1.998 * 32 * 148 * f_mhz * 1e6 / 3 / 1e9), 4)}"})
    prof_path = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(prof_path):
        try:
            with open(prof_path) as f:
                tj = json.load(f)
            roof["traffic"] = tj.get("k_search_dram_bytes_per_launch")
            roof["traffic_source"] = tj.get("source")
        except Exception:
            pass

    # parity (every N) and cpu baseline (N == 1): the oracle on a deterministic sample of the
    # global database against the last timed step's scores (global order)
    cores = cpu_cores()
    budget = args.cpu_budget if world == 1 else min(args.cpu_budget, 8.0)
    idx, res, off, desc = oracle_sample(qs, lens_all, seed, budget, cores)
    ts, ref = run_oracle_step(qs, W, rho, sigma, res, off, cores)
    ref = np.stack(ref)
    mism = int((step_scores[:, idx] != ref).sum())
    if auto_scores is not None:
        mism += int((auto_scores[:, idx] != ref).sum())
    parity = {"checked": int(ref.size) * (2 if auto_scores is not None else 1), "mismatches": mism,
              "sample": desc, "against": "CPU oracle (oracle/sw_oracle.c, Eq.(1) int32)",
              "outputs": "device scores of the last timed step" + (" and of the automatic-threshold step"
                                                                    if auto_scores is not None else "")
              + " in global order",
              "host_api_equal": local_bad_ranks == 0,
              "host_api_note": "sw_search_batch (e2e) and sw_search_stream outputs == the device step's, every rank"}
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        c1 = gen.config("C1")
        t1 = time.perf_counter()
        import oracle
        oracle.scores(c1.queries[0], MATRICES["BLOSUM62"], 10, 2, c1.db.residues, c1.db.offsets, threads=1)
        t1 = time.perf_counter() - t1
        cpu = {"value": round(cells_of(qs, int(off[-1])) / ts / 1e9, 4), "unit": "GCUPS", "cores": cores,
               "cpu_model": cpu_model(), "kind": "oracle", "sample": desc, "seconds": round(ts, 2),
               "single_core_c1": {"value": round(cells_of(c1.queries, c1.db.total_residues) / t1 / 1e9, 4),
                                  "unit": "GCUPS", "seconds": round(t1, 2),
                                  "workload": "C1 in full (20k seqs, query 144), 1 thread"}}

    line = {
        "metric": "GCUPS", "value": round(gcups, 2), "unit": "GCUPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(1e3 * step_s, 3), "higher_is_better": True,
        "scaling": SCALING.get(args.config, "weak"), "vs_baseline": None, "dtype": "s16x2 (int32 recompute)",
        "data": "synthetic",
        "config": {"workload": f"{args.config}: {DB_DESC.get(args.config, 'synthetic DB')}, "
                               f"{n_local} seqs / {db.total_residues / 1e6:.1f}M residues per GPU, "
                               f"queries {[int(q.size) for q in qs]}", "matrix": mat, "gap_open": rho,
                   "gap_extend": sigma, "threshold": T, "seqs_per_gpu": n_local, "seqs_total": n_total,
                   "residues_per_gpu": db.total_residues, "cells_per_step": cells_total,
                   "l2": (f"inputs larger than L2 (device DB ~{2 * db.total_residues / 1e6:.0f} MB > 126 MB)"
                          if 2 * db.total_residues > 126e6 else
                          f"device DB ~{2 * db.total_residues / 1e6:.0f} MB fits in L2 (small config)"),
                   "parallelism": f"db-shard x{world}",
                   **({"c5_shards": max(world, int(os.environ.get("C5_SHARDS", "64")))} if args.config == "C5" else {})},
        "clocks": clk,
        "e2e": {"value": round(e2e_gcups, 2), "unit": "GCUPS", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "api": "sw_search_batch (blocking; queries from host memory, scores copied per query as it finishes into a pinned host buffer reused across steps; DB resident as in PAPER.md L32)"},
        "gpu_launches": int(st["launches"]) * args.steps,
        "roofline": roof,
        "parity": parity,
        "cpu_baseline": cpu,
        "dist": dist_info,
        "regimes": {"long_seqs": st["long_seqs"] // max(1, nq), "short_seqs": st["short_seqs"] // max(1, nq),
                    "recomputed_s32": st["recomputed_s32"], "recompute_ms": round(rec_ms, 3)},
        "stream_db": stream_db,
        "auto_threshold": ({"value": round(cells_total / (auto_ms / 1e3 / args.steps) / 1e9, 2),
                            "ms_per_step": round(auto_ms / args.steps, 3), "unit": "GCUPS"}
                           if auto_ms else None),
        "paper_context": PAPER_CONTEXT,
    }
    print(json.dumps(line), flush=True)
    sw.close()
    if dist_on:
        dist.destroy_process_group()
    if mism or local_bad_ranks:
        print(f"PARITY FAILURE: {mism} oracle mismatches, {local_bad_ranks} ranks with host-API differences",
              file=sys.stderr, flush=True)
        sys.exit(3)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C2")
    ap.add_argument("--threshold", default=None, help="length threshold T (default: the config's, 3072); 'auto' = SW_AUTO_THRESHOLD")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-auto", action="store_true", help="skip the extra automatic-threshold pass")
    ap.add_argument("--no-stream", action="store_true", help="skip the streamed-database (sw_search_stream) pass")
    args = ap.parse_args()
    rank = _env_int("RANK", 0)
    world = _env_int("WORLD_SIZE", 1)
    local_rank = _env_int("LOCAL_RANK", 0)
    if args.impl == "reference":
        bench_reference(args, rank, world)
        return
    bench_ours(args, rank, world, local_rank)


if __name__ == "__main__":
    main()
