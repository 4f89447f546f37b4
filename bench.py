"""bench.py -- SCC detection throughput of the B200-native ECL-SCC path.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` prints ONE JSON line.
A "step" is one whole ECL-SCC run (CSC build, trim, every outer iteration, labels) over
the BASELINE.json workload: at N=1 the 16M-vertex directed mesh sweep graph (configs[3],
"large directed mesh, 16M vertices"), inputs resident in HBM.  Metric: SCC detection
Medges/s = nnz / device time / 1e6 (BASELINE.json), plus Mvertices/s (the paper's unit,
P:208).  For N>1 the same graph is edge-partitioned over the ranks (ecl_scc_partitioned,
strong scaling); ``--config c5`` splits the 64-graph batch over the ranks (weak scaling,
no collective on the data path).  Without WORLD_SIZE in the environment, ``--gpus N > 1``
re-launches this script under ``torch.distributed.run`` with N local ranks.

Every measured configuration is checked bit-exactly against the Tarjan labels that the
cpu_baseline leg computes (the paper verifies every run against Tarjan); a mismatch
raises.  ``ms_per_step`` is the median over the timed steps.

``--impl reference`` times the CPU oracle (iterative Tarjan + max relabel, oracle/) on the
same graph on the host -- the reference arm of this tier (there is no installable
reference implementation: the paper ships no code).
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    "c4": "large directed mesh, 16M vertices, single graph edge-partitioned across 1/2/4/8 GPUs",
    "c5": "batch of 64 mesh sweep graphs (one per discrete-ordinates angle), 2M vertices each, split across 8 GPUs",
    "c2": "directed 3-D tetrahedral-style mesh sweep graph, 1M vertices, degree~4, many small SCCs",
    "c3": "R-MAT power-law graph scale 22 (4M vertices, 64M edges), one giant SCC",
}
L2_NOTE = "flushed between steps (256 MiB write)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c4", choices=sorted(CONFIGS))
    ap.add_argument("--order", default="blocked8", choices=["lex", "blocked8"])
    ap.add_argument("--flags", type=lambda x: int(x, 0), default=0, help="extra ECL_SCC_* plan flags (ablation)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


def dist_env():
    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def spawn(args) -> int:
    """--gpus N > 1 without a launcher: re-run under torch.distributed.run, N local ranks."""
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def load_graph(args, world: int, rank: int):
    import gen
    if args.config in ("c2", "c4"):
        return gen.config(args.config, order=args.order)
    if args.config == "c5":
        from paper_conf_sc_alabandisbb23_b200.dist import split_batch
        return [gen.config("c5one", order=args.order, d=d) for d in split_batch(64, world, rank)]
    return gen.config(args.config)


class Batch:
    """A rank's share of the C5 batch (per-graph CSRs)."""

    def __init__(self, graphs):
        self.graphs = graphs
        self.n = sum(g.n for g in graphs)
        self.nnz = sum(g.nnz for g in graphs)
        self.name = f"{len(graphs)} meshes N=70"


def workload(args, g, world: int, batch: bool):
    w = {"workload": CONFIGS[args.config], "config": args.config, "n": g.n, "nnz": g.nnz,
         "generator": g.name, "seed": {"c2": 2, "c3": 3, "c4": 4, "c5": "5+d"}[args.config],
         "parallelism": (f"batch split x{world}" if batch else
                         f"edge-partitioned x{world}" if world > 1 else "single GPU"),
         "l2": L2_NOTE}
    if args.config in ("c2", "c4", "c5"):
        w["element_order"] = args.order
    if args.flags:
        w["flags"] = hex(args.flags)
    return w


# ------------------------------------------------------------------ clocks sampler
class Clocks:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.samples, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        self.thread.join(timeout=2)
        sm = [float(s[0]) for s in self.samples if len(s) >= 8 and s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if len(s) >= 8 and s[1].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for s in self.samples:
            if len(s) < 8:
                continue
            for k, nm in enumerate(names):
                if s[4 + k].lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ CPU oracle leg
def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def cpu_baseline_leg(graphs, reps: int):
    """The oracle (O1: iterative Tarjan + max relabel) on the same graphs, on the host.

    One graph: one thread, median of `reps` runs (SURVEY 8(d) "one core").  Several graphs
    (C5): one graph per worker thread over all host cores (the oracle is a C library called
    through ctypes, which releases the GIL), the batch timed as a whole ("parallel CPU",
    P:212).  Returns (seconds per pass over all graphs, threads used, labels per graph); the
    labels double as the bench's bit-exact check of the measured configuration."""
    import oracle
    oracle.build()
    if len(graphs) == 1:
        g = graphs[0]
        ts, lab = [], None
        for _ in range(reps):
            t0 = time.perf_counter()
            lab = oracle.tarjan_labels(g.row_ptr, g.col_idx)
            ts.append(time.perf_counter() - t0)
        return statistics.median(ts), 1, [lab]
    cores = max(1, min(len(graphs), os.cpu_count() or 1))
    ts, labs = [], None
    with ThreadPoolExecutor(max_workers=cores) as ex:
        for _ in range(reps):
            t0 = time.perf_counter()
            labs = list(ex.map(lambda h: oracle.tarjan_labels(h.row_ptr, h.col_idx), graphs))
            ts.append(time.perf_counter() - t0)
    return statistics.median(ts), cores, labs


def verify(graphs, gpu_labels, truth):
    """Bit-exact labels of the measured configuration vs Tarjan; raises on any mismatch."""
    import numpy as np
    for k, (g, L, T) in enumerate(zip(graphs, gpu_labels, truth)):
        if L.shape != T.shape or not np.array_equal(L, T):
            bad = int((L != T).sum()) if L.shape == T.shape else -1
            raise RuntimeError(f"bench: GPU labels differ from the Tarjan oracle on graph {k} ({g.name}): "
                               f"{bad} of {g.n} vertices")


def reference_arm(args):
    """Reference arm: the oracle (O1, iterative Tarjan + max relabel) on the same workload,
    each step one full SCC decomposition on the host (C5: all graphs, all host cores)."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    g = load_graph(args, 1, 0)
    graphs = g if isinstance(g, list) else [g]
    batch = isinstance(g, list)
    if batch:
        g = Batch(g)
    for _ in range(args.warmup):
        cpu_baseline_leg(graphs, 1)
    ts = []
    for _ in range(args.steps):
        t, cores, _ = cpu_baseline_leg(graphs, 1)
        ts.append(t)
    t = statistics.median(ts)
    v = g.nnz / t / 1e6
    cfg = workload(args, g, args.gpus, batch)
    cfg["mvertices_per_s"] = round(g.n / t / 1e6, 3)
    sample = (f"full workload ({g.n} vertices, {g.nnz} edges), O1 Tarjan+max-relabel, "
              + (f"one graph per thread on {cores} of {os.cpu_count()} host threads" if batch
                 else f"1 of {os.cpu_count()} host threads") + f" ({cpu_model()})")
    line = {"impl": "reference", "metric": "SCC detection Medges/s", "value": round(v, 3), "unit": "Medges/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
            "higher_is_better": True, "scaling": "weak" if batch else "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic", "config": cfg,
            "cpu_baseline": {"value": round(v, 3), "unit": "Medges/s", "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": round(v, 3), "unit": "Medges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def roofline_traffic(key: str, kernel: str):
    """DRAM bytes per launch of the dominant kernel from the committed ncu capture OF THIS
    CONFIG (profiles/ncu_summary.json, keyed "config/order"); None when there is none."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))["configs"][key]
        k = d["kernels"][kernel]
        return k["dram_bytes_per_launch"], d.get("source")
    except Exception:
        return None, None


def measured_peak():
    try:
        d = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def flush_l2(buf):
    buf.add_(1)     # writes 256 MiB > 126 MB L2


def ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_sc_alabandisbb23_b200 as E

    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    g = load_graph(args, world, rank)
    dev = torch.device("cuda", local)
    flush = torch.zeros(64 * 1024 * 1024, dtype=torch.int32, device=dev)
    batch = None
    if isinstance(g, list):                       # C5: this rank's graphs, batched on its GPU
        batch = g
        g = Batch(batch)
    graphs = batch if batch is not None else [g]
    flags = args.flags | E.NO_VALIDATE
    comm = None

    if batch is not None:
        dgraphs = [(torch.from_numpy(h.row_ptr).to(dev), torch.from_numpy(h.col_idx).to(dev)) for h in batch]
        labs = [torch.empty(h.n, dtype=torch.int32, device=dev) for h in batch]
        plan = E.Plan(g.n, g.nnz, flags)
        plan_t = E.Plan(g.n, g.nnz, flags | E.TIME_STAGES)

        def step(p=plan):
            return E.ecl_scc_batched(dgraphs, labs, plan=p, stats=True)[1]
    elif world == 1:
        rp = torch.from_numpy(g.row_ptr).to(dev)
        ci = torch.from_numpy(g.col_idx).to(dev)
        labs = [torch.empty(g.n, dtype=torch.int32, device=dev)]
        plan = E.Plan(g.n, g.nnz, flags)
        plan_t = E.Plan(g.n, g.nnz, flags | E.TIME_STAGES)

        def step(p=plan):
            return E.ecl_scc(rp, ci, labs[0], plan=p, stats=True)[1]
    else:
        bounds = E.ecl_scc_partition_rows(world, g.row_ptr)
        rb, re_ = bounds[rank], bounds[rank + 1]
        lrp = torch.from_numpy((g.row_ptr[rb:re_ + 1] - g.row_ptr[rb]).astype(np.int32)).to(dev)
        lci = torch.from_numpy(g.col_idx[g.row_ptr[rb]:g.row_ptr[re_]]).to(dev)
        labs = [torch.empty(g.n, dtype=torch.int32, device=dev)]
        uid = [E.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        comm = E.Comm(world, rank, uid[0])
        pplan = E.PartPlan(comm, g.n, rb, re_, lci.numel(), flags)
        plan_t = None

        def step(p=None):
            return E.ecl_scc_partitioned(comm, g.n, rb, re_, lrp, lci, labs[0], plan=pplan, stats=True)[1]

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    got = [l.cpu().numpy() for l in labs]

    clocks = Clocks(local)
    clocks.start()
    times, stats_all = [], []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for _ in range(args.steps):
        flush_l2(flush)
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        stats_all.append(step())
        b.record()
        b.synchronize()
        times.append(a.elapsed_time(b))
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    stats = stats_all[-1]
    # stage breakdown + roofline figures, same workload, stage events on
    rstats = []
    if plan_t is not None:
        step(plan_t)                              # first use allocates the tile packs: untimed
        for _ in range(max(3, min(args.steps, 5))):
            flush_l2(flush)
            rstats.append(step(plan_t))
    ck = clocks.stop()
    t_ms = statistics.median(times)
    if world > 1:
        tt = torch.tensor([t_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_ms = float(tt.item())

    # ---- end to end through the public API with host buffers (pinned H2D + D2H)
    e2e = None
    if not args.no_e2e and world == 1 and batch is None:
        hrp = torch.from_numpy(g.row_ptr).pin_memory()
        hci = torch.from_numpy(g.col_idx).pin_memory()
        hlab = torch.empty(g.n, dtype=torch.int32).pin_memory()
        et = []
        for k in range(args.warmup + args.steps):
            flush_l2(flush)
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record()
            E.ecl_scc_host(hrp, hci, hlab, plan=plan)   # C ABI with host buffers: H2D, run, D2H
            b.record()
            b.synchronize()
            if k >= args.warmup:
                et.append(a.elapsed_time(b))
        te = statistics.median(et)
        if not np.array_equal(hlab.numpy(), got[0]):
            raise RuntimeError("bench: ecl_scc_host labels differ from ecl_scc's")
        e2e = {"value": round(g.nnz / te / 1e3, 3), "unit": "Medges/s", "ms_per_step": round(te, 3),
               "h2d_bytes_per_step": int(hrp.numel() * 4 + hci.numel() * 4),
               "d2h_bytes_per_step": int(hlab.numel() * 4)}
    elif not args.no_e2e and batch is not None:
        # C5: this rank's batch through ecl_scc_batched_host (pinned CSRs in, labels out)
        hg = [(torch.from_numpy(h.row_ptr).pin_memory(), torch.from_numpy(h.col_idx).pin_memory()) for h in batch]
        hl = [torch.empty(h.n, dtype=torch.int32).pin_memory() for h in batch]
        et = []
        for k in range(args.warmup + args.steps):
            flush_l2(flush)
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record()
            E.ecl_scc_batched_host(hg, hl, plan=plan)   # C ABI with host buffers: H2D, run, D2H
            b.record()
            b.synchronize()
            if k >= args.warmup:
                et.append(a.elapsed_time(b))
        te = statistics.median(et)
        for l, ref in zip(hl, got):
            if not np.array_equal(l.numpy(), ref):
                raise RuntimeError("bench: ecl_scc_batched_host labels differ from ecl_scc_batched's")
        ebytes = torch.tensor([te, sum(x.numel() + y.numel() for x, y in hg) * 4, sum(l.numel() for l in hl) * 4],
                              dtype=torch.float64, device=dev)
        if world > 1:                                   # whole job: slowest rank, all ranks' bytes
            tmax = ebytes[:1].clone()
            dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
            dist.all_reduce(ebytes, op=dist.ReduceOp.SUM)
            ebytes[0] = tmax[0]
        te = float(ebytes[0].item())
        e2e = {"value": None, "unit": "Medges/s", "ms_per_step": round(te, 3),
               "h2d_bytes_per_step": int(ebytes[1].item()), "d2h_bytes_per_step": int(ebytes[2].item())}

    # ---- bit-exact check of the measured configuration against the oracle's labels (the
    # cpu_baseline leg): every rank checks its own graphs (C4 partitioned: rank 0 the whole)
    cpu = None
    if rank == 0 or batch is not None:
        reps = 3 if batch is None else 1
        tc, cores, truth = cpu_baseline_leg(graphs, reps)
        verify(graphs, got, truth)
        if world == 1 and not args.no_cpu_baseline:
            sample = (f"full workload ({g.n} vertices, {g.nnz} edges), O1 iterative Tarjan + max relabel, "
                      + (f"median of {reps}, 1 of {os.cpu_count()} host threads" if batch is None else
                         f"one graph per thread on {cores} of {os.cpu_count()} host threads")
                      + f" ({cpu_model()})")
            cpu = {"value": round(g.nnz / tc / 1e6, 3), "unit": "Medges/s", "cores": cores, "kind": "oracle",
                   "sample": sample}

    total_nnz, total_n = g.nnz, g.n
    if batch is not None and world > 1:             # weak scaling: every rank's graphs count
        tt = torch.tensor([g.nnz, g.n], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.SUM)
        total_nnz, total_n = int(tt[0].item()), int(tt[1].item())
    comm_ms = None
    if world > 1 and batch is None:
        cm = torch.tensor([statistics.median(s["ms_comm"] for s in stats_all)], dtype=torch.float64, device=dev)
        dist.all_reduce(cm, op=dist.ReduceOp.MAX)
        comm_ms = float(cm.item())
    if rank != 0:
        if comm is not None:
            comm.close()
        dist.destroy_process_group() if world > 1 else None
        return 0

    value = total_nnz / t_ms / 1e3  # Medges/s of the whole job
    if e2e is not None and e2e["value"] is None:
        e2e["value"] = round(total_nnz / e2e["ms_per_step"] / 1e3, 3)
    peak, peak_src = measured_peak()
    roof = None
    if rstats:
        pb = statistics.median(s["prop_bytes"] for s in rstats)
        pms = statistics.median(s["ms_prop"] for s in rstats)
        achieved = pb / (pms * 1e-3) / 1e9 if pms > 0 else None
        # the dominant kernel: k_prop_async (one persistent launch per outer iteration) on
        # graphs without long rows, the pass kernels k_prop_tile + k_prop_heavy otherwise
        async_path = args.config != "c3"
        kname = "k_prop_async" if async_path else "k_prop_tile"
        key = args.config + (f"/{args.order}" if args.config != "c3" else "")
        traffic, tsrc = roofline_traffic(key, kname)
        iters = statistics.median(s["iterations"] for s in rstats)
        roof = {"bound": "hbm",
                "kernel": ("Phase 2 (k_prop_async; tile packs written by the compaction scatter)" if async_path
                           else "Phase 2 (k_prop_tile + k_prop_heavy)"),
                "algorithmic_bytes_per_launch": int(pb / iters) if async_path and iters else None,
                "achieved": round(achieved, 1) if achieved else None, "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4) if achieved else None,
                "traffic": traffic, "traffic_source": tsrc, "peak_source": peak_src,
                "algorithmic_bytes_per_step": int(pb), "prop_ms_per_step": round(pms, 3),
                "passes_per_step": statistics.median(s["passes"] for s in rstats),
                "stage_ms": {k: round(statistics.median(s[k] for s in rstats), 3)
                             for k in ("ms_ingest", "ms_compact", "ms_prop")}}
    cfg = workload(args, g, world, batch is not None)
    cfg["mvertices_per_s"] = round(total_n / t_ms / 1e3, 3)
    if batch is not None and world > 1:
        cfg["n_total"], cfg["nnz_total"] = total_n, total_nnz
    line = {
        "metric": "SCC detection Medges/s", "value": round(value, 3), "unit": "Medges/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t_ms, 4),
        "ms_mean": round(statistics.fmean(times), 4),
        "higher_is_better": True, "scaling": "weak" if batch is not None else "strong", "vs_baseline": None,
        "dtype": "int32", "data": "synthetic", "config": cfg,
        "verified": "labels bit-exact vs the Tarjan oracle (every graph of this rank's share)",
        "gpu_launches": int(sum(s["kernel_launches"] for s in stats_all)),
        "iterations": stats["iterations"], "passes": stats["passes"],
        "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": ck,
    }
    if comm_ms is not None:
        info = comm.info()
        line["comm"] = {"ms_per_step": round(comm_ms, 4), "share": round(comm_ms / t_ms, 4),
                        "bytes_per_step_rank0": int(stats["comm_bytes"]), "exchanges": int(stats["exchanges"]),
                        "halo_exchange": ("fused: multimem.red.max (NVLS)" if info["multimem"] else
                                          "fused: remote atomicMax over NVLink peers" if info["device_api"] else
                                          "ncclAllReduce(MAX) of the halo"),
                        "note": "ms_per_step: the collectives (barriers, degree / count / label all-reduces); "
                                "the fused halo pushes run inside k_prop_async"}
    print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        return spawn(args)
    if args.impl == "reference":
        return reference_arm(args)
    return ours(args)


if __name__ == "__main__":
    sys.exit(main())
