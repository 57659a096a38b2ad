"""Debug: GPU vs oracle error as a function of iteration count (C1)."""
import sys, numpy as np
sys.path.insert(0, ".")
from oracle import runner as R
from sf_inputs import data as D, graphs as G
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime

def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))

g = G.mlp_train()
st, ds = D.init_state(g), D.datasets(g)
for iters in (1, 2, 3, 5, 10, 20, 50, 100):
    with Runtime([0]) as rt:
        gh = rt.register(g); gh.partition(); gh.bind(0, host_staging=True); gh.load(0, {**st, **ds})
        j = rt.start_training(gh, 0, iters, -1); rt.wait_job(j, 60)
        got = {i: gh.read(0, i) for i in st}
        acts = {n: gh.read(0, g.tid(n)) for n in ("x", "z1", "h1", "logits", "loss", "dl", "dW2", "dW1", "db1", "dh1")}
    ref = R.run(g, iters, st, ds, keep_stagings=False)
    errs = {g.tensors[i].name: rel(got[i], ref.state[i]) for i in st if st[i].dtype == np.float32}
    print(iters, "step", got[g.tid("step")].ravel(), ref.state[g.tid("step")].ravel(), {k: f"{v:.1e}" for k, v in errs.items()})
    if iters == 1:
        # recompute iteration-1 activations with the oracle to localize
        from oracle import ops as O
        T = {**{i: a.copy() for i, a in st.items()}, **ds}
        shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
        for op in g.ops:
            if op.type in (7, 10):
                continue
            O.apply_op(op, T, shapes)
        for n, a in acts.items():
            print("  ", n, f"{rel(a, T[g.tid(n)]):.2e}")
