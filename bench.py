"""Benchmark: full two-stage FP64 tridiagonalization (DBBR + GPU bulge chasing) on B200.

Metric (BASELINE.json): FP64 TFLOPs = (4 n^3 / 3) / (t_SBR + t_BC), n = 32768 headline (configs[2],
b = 64, nb = 16, k = 1024), with the SBR/BC time split.  One "step" = restore A from a resident
copy (D2D, 8.6 GB, included in the step time) + trid_sytrd_2stage (both stages, Q reflectors stored).
Inputs live in HBM before the timed region; the 8.6 GB matrix is far larger than the 126 MB L2, so no
explicit flush is needed between steps.

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--n N --b B ...]
Multi-GPU (torchrun): stage 1 is sharded over the ranks (block-cyclic column blocks, per-panel NCCL
broadcast + all-reduce), the band is gathered to rank 0 and stage 2 runs there; the
matrix is the same for every N (strong scaling); time is the max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAK_FP64_DMMA_TFLOPS = 37.0     # measured: profiles/r01_fp64_microbench.jsonl (DMMA m16n8k8, 1965 MHz)
CONFIGS = {
    "n256": dict(n=256, b=32, nb=8, k=256, seed=1001, desc="n=256 random symmetric FP64, b=32, nb=8"),
    "n8192": dict(n=8192, b=64, nb=16, k=1024, seed=2001, desc="n=8192 random symmetric FP64, b=64, nb=16"),
    "n32768": dict(n=32768, b=64, nb=16, k=1024, seed=3001,
                   desc="n=32768 random symmetric FP64, b=64, nb=16, k=1024 on 1xB200"),
    "n32768b128": dict(n=32768, b=128, nb=16, k=1024, seed=3001,
                       desc="n=32768 random symmetric FP64, b=128, nb=16, k=1024 on 1xB200"),
    "n49152": dict(n=49152, b=64, nb=16, k=1024, seed=4001, kind="clusters",
                   desc="n=49152 clustered-spectrum symmetric FP64 (32 clusters), b=64, nb=16, k=1024"),
    **{f"n16384b{bb}": dict(n=16384, b=bb, nb=min(16, bb), k=1024, seed=5001,
                            desc=f"n=16384 random symmetric FP64, b={bb}, nb={min(16, bb)}, k=1024 (band sweep)")
       for bb in (32, 64, 128, 256)},
}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p.get("hbm_gbs", 6549.4)), "measured"
    except Exception:
        return 6650.0, "fallback"


# ------------------------------------------------------------------ algorithmic work (pure counting)
def dbbr_flops(n, b, k, fold=True):
    """Per-class algorithmic flops of the DBBR loop structure (same loop bounds as Alg. 1 / R4).  fold: the Z
    builder's corrections X -= Y_< U1 + Z_< U2 (4 m kk ncols flops, R4e) run inside the SYMM launch (the
    single-GPU default, TRID_ZY_FOLD) and count towards its class."""
    fl = {"symm": 0.0, "syr2k": 0.0, "symm_launches": 0, "syr2k_launches": 0}
    i = 0
    while i + b + 1 < n:
        ncols, j, jlast = 0, i, i
        while j < i + k and j + b + 1 < n:
            m = n - j - b
            kk = min(b, m)
            fl["symm"] += 2.0 * m * m * kk + (4.0 * m * kk * ncols if fold else 0.0)
            fl["symm_launches"] += 1
            ncols += kk
            jlast = j
            j += b
        e = jlast + b
        if e < n:
            M = n - e
            fl["syr2k"] += 2.0 * M * (M + 1) * ncols
            fl["syr2k_launches"] += 1
        i += k
    return fl


def bc_bytes(n, b):
    """Algorithmic bytes of the chase: per step read+write of the lower triangle of D_m,
    read+write of O_m, and the write of v: 8 (2 L(L+1)/2 + 2 L2 L + L)."""
    import numpy as np
    if b < 2 or n < 3:
        return 0.0
    total = 0.0
    s = np.arange(0, n - 2, dtype=np.int64)
    nst = (n - 3 - s) // b + 1
    mmax = int(nst.max())
    for m in range(mmax):
        sel = s[nst > m]
        r0 = sel + 1 + m * b
        r1 = np.minimum(sel + (m + 1) * b, n - 1)
        L = r1 - r0 + 1
        L2 = np.minimum(r1 + b, n - 1) - r1
        total += float(np.sum(8.0 * (L * (L + 1) + 2 * L2 * L + L)))
    return total


# ------------------------------------------------------------------ clocks
class Clocks:
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,power.draw")

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        self.rows = []
        if self.p is None:
            return
        self.p.terminate()
        out = self.p.communicate()[0]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 7 and f[0].replace(".", "").isdigit():
                self.rows.append(f)

    def summary(self):
        if not getattr(self, "rows", None):
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows]
        mx = max(float(r[1]) for r in self.rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(sm), "power_w_max": max(float(r[6]) for r in self.rows if r[6] not in ("[N/A]",))}


# ------------------------------------------------------------------ CPU oracle timing (test infra)
def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def oracle_worker(n, b, seed, kind, variant):
    """One oracle run in this process (a replica of the all-cores measurement); prints its seconds."""
    import oracle
    import trid_gen
    A = trid_gen.random_symmetric_np(n, seed)
    print(json.dumps({"seconds": oracle.timed_run(kind, A, b, variant)}))
    return 0


def oracle_replicas(n, b, seed, kind, variant, procs):
    """procs concurrent single-threaded oracle processes (one per host core): the oracle as it stands on all
    cores, without changing its code.  Returns (wall seconds, per-process seconds)."""
    cmd = [sys.executable, os.path.abspath(__file__), "--oracle-worker", str(n), str(b), str(seed), kind, variant]
    t0 = time.perf_counter()
    ps = [subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True) for _ in range(procs)]
    secs = []
    for p in ps:
        out = p.communicate()[0]
        try:
            secs.append(json.loads(out.strip().splitlines()[-1])["seconds"])
        except Exception:
            pass
    return time.perf_counter() - t0, secs


def cpu_baseline(b, seed, sizes=(768, 1024, 1536), n_all=1536, n_target=32768):
    """the CPU oracle (O1 = unblocked dsytd2; O2 = naive SBR + naive bulge chase, vectors stored)
    timed on this host: single-threaded at several n with gcc -O3 -march=native (and -O2 at the smallest n),
    all cores (one single-threaded replica per core) at n_all, and a c n^3 fit of O2 extrapolated to n_target
    (labelled "extrapolated").  The headline value is the all-cores O2 throughput at n_all."""
    import oracle
    import trid_gen
    oracle.build()
    oracle.build(variant="O3native")
    cores = os.cpu_count() or 1
    runs = []
    for n in sizes:
        A = trid_gen.random_symmetric_np(n, seed)
        for kind in ("O1", "O2"):
            for variant in (("O2", "O3native") if n == sizes[0] else ("O3native",)):
                t = oracle.timed_run(kind, A, b, variant)
                runs.append({"kind": kind, "flags": variant, "n": n, "threads": 1, "seconds": round(t, 3),
                             "tflops": round(4.0 * n ** 3 / 3.0 / t / 1e12, 6)})
    pts = [(r["n"], r["seconds"]) for r in runs if r["kind"] == "O2" and r["flags"] == "O3native"]
    c = sum(t / n ** 3 for n, t in pts[-2:]) / len(pts[-2:])
    wall, secs = oracle_replicas(n_all, b, seed, "O2", "O3native", cores)
    flop_all = 4.0 * n_all ** 3 / 3.0 * len(secs)
    value = flop_all / max(max(secs) if secs else wall, 1e-9) / 1e12
    runs.append({"kind": "O2", "flags": "O3native", "n": n_all, "threads": cores, "replicas": len(secs),
                 "seconds_max": round(max(secs), 3) if secs else None, "wall": round(wall, 3),
                 "tflops": round(value, 6)})
    t_ext = c * n_target ** 3
    return {"value": round(value, 6), "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
            "sample": f"oracle O2 (naive SBR O2a + naive bulge chase O2b, vectors stored, C, gcc -O3 -march=native) "
                      f"at n={n_all}, b={b}, seed {seed}, {len(secs)} single-threaded replicas on {cores} host cores; "
                      f"same 4n^3/3 flop convention",
            "cpu_model": cpu_model(), "runs": runs,
            "extrapolated": {"n": n_target, "label": "extrapolated", "fit": "c*n^3 from the two largest "
                             "single-threaded O2 -O3 points", "seconds_1core": round(t_ext, 1),
                             "seconds_all_cores": round(t_ext / max(cores, 1), 1),
                             "tflops_1core": round(4.0 * n_target ** 3 / 3.0 / t_ext / 1e12, 6)}}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


METRIC = "FP64 TFLOPs (4n^3/3) full tridiag at n=32768, SBR/BC time split, 1/2/4/8 GPU"   # BASELINE.json


def run_reference(args):
    """The reference arm: this tier has no reference implementation (the paper only), so the CPU oracle as it
    stands is the reference, timed on the host cores (one single-threaded replica per core, each a bounded
    sample of the workload: the same matrix recipe and b at n = --ref-n)."""
    ws, rank, _ = dist_env()
    if rank != 0:
        return 0
    import oracle
    oracle.build(variant="O3native")
    cfg = CONFIGS[args.config]
    n_s = args.ref_n
    cores = os.cpu_count() or 1
    times = []
    nrep = cores
    for i in range(args.warmup + args.steps):
        wall, secs = oracle_replicas(n_s, cfg["b"], cfg["seed"], "O2", "O3native", cores)
        nrep = len(secs) or 1
        if i >= args.warmup:
            times.append(max(secs) if secs else wall)
    t = sum(times)
    value = 4.0 * n_s ** 3 / 3.0 * nrep * args.steps / t / 1e12
    line = {"impl": "reference", "metric": METRIC, "value": round(value, 6),
            "unit": "TFLOP/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1e3 * t / args.steps, 3), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg["desc"], "n": cfg["n"], "b": cfg["b"], "nb": cfg["nb"], "k": cfg["k"],
                       "seed": cfg["seed"], "sample_n": n_s},
            "cpu_baseline": {"value": round(value, 6), "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
                             "cpu_model": cpu_model(),
                             "sample": f"each step = {nrep} concurrent single-threaded CPU oracle runs (naive SBR + "
                                       f"naive BC, gcc -O3 -march=native) at n={n_s}, b={cfg['b']}"},
            "e2e": {"value": round(value, 6), "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def spawn_ranks(args):
    """--gpus N without a launcher: re-run this script under torch.distributed.run with N local ranks."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def dry_run(args):
    """--dry-run: the rank plumbing only (gloo, CPU): every rank reports itself, rank 0 prints the roster."""
    import torch
    import torch.distributed as dist
    ws, rank, local = dist_env()
    if ws > 1:
        dist.init_process_group("gloo")
    t = torch.tensor([rank, local, os.getpid()], dtype=torch.int64)
    rows = [torch.zeros_like(t) for _ in range(ws)]
    if ws > 1:
        dist.all_gather(rows, t)
    else:
        rows = [t]
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": args.gpus, "world_size": ws,
                          "ranks": [r.tolist() for r in rows]}))
    if ws > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="n32768", choices=sorted(CONFIGS))
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--b", type=int, default=0)
    ap.add_argument("--k", type=int, default=-1)
    ap.add_argument("--nb", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--ref-n", type=int, default=1024)
    ap.add_argument("--eig-only", action="store_true", help="eigenvalues-only BC (V2 = NULL)")
    ap.add_argument("--dry-run", action="store_true", help="rank plumbing only (gloo, no GPU work)")
    ap.add_argument("--mode", default="sharded", choices=["sharded", "replicas"],
                    help="N > 1: sharded = one matrix, stage 1 sharded over the ranks (strong scaling); replicas = "
                         "one independent matrix per rank (batched multi-matrix tridiagonalization, weak scaling)")
    ap.add_argument("--oracle-worker", nargs=5, metavar=("N", "B", "SEED", "KIND", "FLAGS"), help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.oracle_worker:
        n_, b_, s_, kind_, var_ = args.oracle_worker
        return oracle_worker(int(n_), int(b_), int(s_), kind_, var_)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return spawn_ranks(args)
    ws_env = int(os.environ.get("WORLD_SIZE", "1"))
    if ws_env != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws_env}", file=sys.stderr)
        return 2
    if args.dry_run:
        return dry_run(args)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_wangdzwzljz25_b200 as trid
    import trid_gen

    ws, rank, local = dist_env()
    if ws > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl")
    dev = torch.device("cuda", local if ws > 1 else 0)
    torch.cuda.set_device(dev)
    cfg = dict(CONFIGS[args.config])
    if args.n:
        cfg["n"] = args.n
    if args.b:
        cfg["b"] = args.b
    if args.k >= 0:
        cfg["k"] = args.k
    if args.nb:
        cfg["nb"] = args.nb
    n, b, nb, k = cfg["n"], cfg["b"], min(cfg["nb"], cfg["b"]), cfg["k"] or trid.default_k(cfg["n"], cfg["b"])
    if args.n or args.b or args.k >= 0:
        cfg["desc"] = f"n={n} random symmetric FP64, b={b}, nb={nb}, k={k}"

    want = not args.eig_only
    stream = torch.cuda.current_stream()
    sharded = ws > 1 and args.mode == "sharded"
    if not sharded:
        seed = cfg["seed"] + (rank if ws > 1 else 0)   # replicas: an independent matrix per rank
        if cfg.get("kind"):
            A0, _ = trid_gen.clustered_symmetric(n, seed, kind=cfg["kind"], device=dev)
        else:
            A0 = trid_gen.random_symmetric(n, seed, device=dev)
        A = torch.empty_like(A0)
        nbytes, v2len, t2len = trid.sytrd_2stage_bufsize(n, b, nb, k)
        work = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=dev)
        out = (torch.empty(n, dtype=torch.float64, device=dev),
               torch.empty(max(n - 1, 1), dtype=torch.float64, device=dev),
               torch.empty(n, dtype=torch.float64, device=dev),
               torch.empty(max(v2len, 1), dtype=torch.float64, device=dev) if want else None,
               torch.empty(max(t2len, 1), dtype=torch.float64, device=dev) if want else None)

        def run(Ain):
            trid.sytrd_2stage(Ain, b, nb=nb, k=k, want_vectors=want, work=work, out=out)
            return out[0], out[1], out[2]
    else:
        # multi-GPU: stage 1 sharded over the ranks (block-cyclic columns, NCCL per panel), band gathered to
        # rank 0, stage 2 on rank 0 (one chase is one dependency chain).  Same matrix as N = 1: strong scaling.
        comm = trid.comm_nccl()
        cols = trid_gen.block_cyclic_columns(n, b, ws, rank)
        A0 = trid_gen.random_symmetric_rows(n, cfg["seed"], cols, device=dev)
        A = torch.empty_like(A0)
        work = torch.empty(max(trid.sbr_dbbr_mg_bufsize(n, b, nb, k, ws, rank), 256), dtype=torch.uint8, device=dev)
        tau1 = torch.empty(n, dtype=torch.float64, device=dev)
        AB = torch.empty((n, b + 1), dtype=torch.float64, device=dev)
        bc_out = None
        if rank == 0:
            bcb, v2len, t2len = trid.bulge_chase_bufsize(n, b)
            bc_work = torch.empty(max(bcb, 256), dtype=torch.uint8, device=dev)
            bc_out = (torch.empty(n, dtype=torch.float64, device=dev),
                      torch.empty(max(n - 1, 1), dtype=torch.float64, device=dev),
                      torch.empty(max(v2len, 1), dtype=torch.float64, device=dev) if want else None,
                      torch.empty(max(t2len, 1), dtype=torch.float64, device=dev) if want else None)

        def run(Ain):
            trid.sbr_dbbr_mg(comm, Ain, n, b, nb=nb, k=k, tau1=tau1, work=work)
            trid.band_gather(comm, Ain, n, b, root=0, AB=AB)
            if rank == 0:
                trid.bulge_chase_band(AB, n, b, want_vectors=want, work=bc_work, out=bc_out)
                return bc_out[0], bc_out[1], tau1
            return None

    def step():
        A.copy_(A0)
        run(A)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(dev.index) as clk:
        trid.profile_begin()
        l0 = trid.kernel_launches()
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        launches = trid.kernel_launches() - l0
        stages = trid.profile_end()
    ms = ev0.elapsed_time(ev1)
    if ws > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    flop = 4.0 * n ** 3 / 3.0
    nmat = ws if (ws > 1 and not sharded) else 1   # matrices per step over all ranks
    value = nmat * flop * args.steps / (ms * 1e-3) / 1e12   # sharded: one matrix per step (strong scaling)
    per = {c: (v[0] / args.steps, v[1] / args.steps) for c, v in stages.items()}
    t_bc = per["bulge_chase"][0]
    t_sbr = sum(per[c][0] for c in trid.SBR_CLASSES)

    # roofline: the dominant DBBR contraction (largest time share) against the measured FP64 DMMA peak
    fold = not sharded and os.environ.get("TRID_ZY_FOLD", "1")[:1] != "0"
    fl = dbbr_flops(n, b, k, fold=fold)
    cand = {"symm": (fl["symm"], per["symm"]), "syr2k": (fl["syr2k"], per["syr2k"])}
    dom = max(cand, key=lambda c: cand[c][1][0])
    dflops, (dms, dcalls) = cand[dom]
    achieved = (dflops / max(dcalls, 1)) / ((dms / max(dcalls, 1)) * 1e-3) / 1e12 if dcalls else 0.0
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tpath):
        try:
            traffic = json.load(open(tpath)).get(f"{args.config}:{dom}")
        except Exception:
            traffic = None
    bc_traffic = None
    if os.path.exists(tpath):
        try:
            bc_traffic = json.load(open(tpath)).get(f"{args.config}:bulge_chase")
        except Exception:
            bc_traffic = None
    hbm, hbm_kind = peaks()
    bcb = bc_bytes(n, b)
    bc_gbs = bcb / (t_bc * 1e-3) / 1e9 if t_bc > 0 else 0.0

    line = {
        "metric": METRIC,
        "value": round(value, 4), "unit": "TFLOP/s", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(ms / args.steps, 3), "higher_is_better": True, "scaling": "strong" if sharded else "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg["desc"], "n": n, "b": b, "nb": nb, "k": k, "seed": cfg["seed"],
                   "parallelism": (f"sbr-colblock-cyclic-x{ws}+bc-rank0" if sharded else
                                   (f"replicas-x{ws}" if ws > 1 else "single-gpu")),
                   "l2": "inputs larger than L2 (n^2*8 B matrix restored from a resident copy each step)",
                   "vectors": "stored (V1 in A, tau1, V2, tau2)" if want else "eigenvalues-only"},
        "t_sbr_ms": round(t_sbr, 3), "t_bc_ms": round(t_bc, 3),
        "split": {"sbr": round(t_sbr / (t_sbr + t_bc), 4) if t_sbr + t_bc > 0 else None,
                  "bc": round(t_bc / (t_sbr + t_bc), 4) if t_sbr + t_bc > 0 else None},
        "stages_ms_per_step": {c: round(v[0], 3) for c, v in per.items()},
        "stage_calls_per_step": {c: v[1] for c, v in per.items()},
        "roofline": {"bound": "tensor", "kernel": dom, "achieved": round(achieved, 3),
                     "peak": PEAK_FP64_DMMA_TFLOPS, "unit": "TFLOP/s", "frac": round(achieved / PEAK_FP64_DMMA_TFLOPS, 4),
                     "traffic": traffic,
                     "peak_source": "measured FP64 DMMA microbenchmark (profiles/r01_fp64_microbench.jsonl); "
                                    "MEASURED_PEAKS.json has no FP64 figure"},
        "roofline_bc": {"bound": "hbm", "kernel": "bulge_chase", "achieved": round(bc_gbs, 1), "peak": hbm,
                        "unit": "GB/s", "frac": round(bc_gbs / hbm, 4), "traffic": bc_traffic,
                        "algorithmic_bytes": bcb, "peak_source": hbm_kind},
        "sbr_tflops": round(flop / (t_sbr * 1e-3) / 1e12, 3) if t_sbr > 0 else None,
        "gpu_launches": int(launches),
        "clocks": clk.summary(),
    }

    # ---- end to end through the public API with host buffers (pinned H2D of A, D2H of d, e, tau1)
    if not args.no_e2e and args.e2e_steps > 0:
        Ah = torch.empty(A0.shape, dtype=torch.float64, pin_memory=True)
        Ah.copy_(A0)
        dh = torch.empty(n, dtype=torch.float64, pin_memory=True)
        eh = torch.empty(max(n - 1, 1), dtype=torch.float64, pin_memory=True)
        th = torch.empty(n, dtype=torch.float64, pin_memory=True)
        torch.cuda.synchronize()

        def fetch(res):
            if res is not None:
                dh.copy_(res[0], non_blocking=True)
                eh.copy_(res[1][: max(n - 1, 1)], non_blocking=True)
                th.copy_(res[2], non_blocking=True)

        def timed_e2e(pipelined):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            if ws > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0.record(stream)
            if not pipelined:
                for _ in range(args.e2e_steps):
                    A.copy_(Ah, non_blocking=True)
                    fetch(run(A))
            else:
                # serving pipeline: step i+1's H2D (copy stream, into the other device buffer) overlaps step i's
                # compute; every step still copies its whole input from pinned host memory inside the region
                bufs = (A, Abuf2)
                ready = [torch.cuda.Event(), torch.cuda.Event()]
                free = [torch.cuda.Event(), torch.cuda.Event()]
                cs.wait_stream(stream)
                with torch.cuda.stream(cs):
                    bufs[0].copy_(Ah, non_blocking=True)
                    ready[0].record(cs)
                for i in range(args.e2e_steps):
                    cur, nxt = i % 2, (i + 1) % 2
                    if i + 1 < args.e2e_steps:
                        with torch.cuda.stream(cs):
                            if i >= 1:
                                cs.wait_event(free[nxt])
                            bufs[nxt].copy_(Ah, non_blocking=True)
                            ready[nxt].record(cs)
                    stream.wait_event(ready[cur])
                    fetch(run(bufs[cur]))
                    free[cur].record(stream)
            e1.record(stream)
            torch.cuda.synchronize()
            ems = e0.elapsed_time(e1)
            if ws > 1:
                t = torch.tensor([ems], dtype=torch.float64, device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ems = float(t.item())
            return nmat * flop * args.e2e_steps / (ems * 1e-3) / 1e12

        Abuf2 = torch.empty_like(A) if not sharded else None
        cs = torch.cuda.Stream(device=dev)   # the copy stream of the pipelined mode (created outside the timing)
        serial = timed_e2e(False)
        piped = None
        if not sharded:
            timed_e2e(True)   # untimed warm-up of the pipelined path (second buffer, copy stream, events)
            piped = timed_e2e(True)
        line["e2e"] = {"value": round(piped if piped is not None else serial, 4), "unit": "TFLOP/s",
                       "h2d_bytes_per_step": 8 * A0.numel() * ws, "d2h_bytes_per_step": 8 * (n + (n - 1) + n) * nmat,
                       "steps": args.e2e_steps,
                       "mode": ("pipelined: step i+1's pinned H2D on a copy stream overlaps step i's compute "
                                "(double-buffered device input)") if piped is not None else "serial",
                       "serial_value": round(serial, 4),
                       "note": "V1/V2 reflectors stay device-resident for the back transformation"}
        del Ah, Abuf2
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(b, cfg["seed"])
    if rank == 0:
        print(json.dumps(line))
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
