"""Quick device timing of ecl_scc on the BASELINE configs (development helper)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
import paper_conf_sc_alabandisbb23_b200 as E

def run(name, g, flags=0, reps=5):
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    plan = E.Plan(g.n, g.nnz, flags)
    lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
    _, st = E.ecl_scc(rp, ci, lab, plan=plan, stats=True)
    ts = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); E.ecl_scc(rp, ci, lab, plan=plan); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    t = float(np.median(ts))
    cnt = plan.counters()[:4]
    print(f"{name:28s} flags={flags} prof={cnt} n={g.n} m={g.nnz} t={t:.3f} ms  {g.nnz/t/1e3:.1f} Me/s  iters={st['iterations']} passes={st['passes']} per-iter={st['passes_iter'][:8]} ein={st['edges_in'][:6]}", flush=True)

FLAGS = [int(x) for x in os.environ.get('QT_FLAGS', '0,32,64,96').split(',')]

if __name__ == "__main__":
    which = sys.argv[1:] or ["c2", "c4", "c3"]
    for w in which:
        if w == "c2":
            for order in ("lex", "blocked8"):
                g = gen.config("c2", order=order)
                for fl in FLAGS: run(f"c2 {order}", g, fl)
        elif w == "c4":
            for order in ("lex", "blocked8"):
                g = gen.config("c4", order=order)
                for fl in FLAGS: run(f"c4 {order}", g, fl, reps=3)
        elif w == "c3":
            g = gen.config("c3")
            for fl in (0, E.IDENTITY_IDS): run("c3 rmat22", g, fl)
        elif w == "c1":
            run("c1", gen.config("c1"))
