"""Debug only: one-step GPU vs oracle started from the GPU's state (localizes a bad step)."""
import sys, numpy as np
sys.path.insert(0, ".")
from oracle import runner as R, ops as O
from sf_inputs import data as D, graphs as G
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime

def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))

g = G.mlp_train()
st, ds = D.init_state(g), D.datasets(g)
shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
state = {i: a.copy() for i, a in st.items()}
names = ("z1", "h1", "logits", "loss", "dl", "dW2", "db2", "dh1", "dz1", "db1", "dW1")
with Runtime([0]) as rt:
    gh = rt.register(g); gh.partition(); gh.bind(0, host_staging=True); gh.load(0, ds)
    worst = 0
    for it in range(60):
        gh.load(0, state)
        j = rt.start_training(gh, 0, 1, -1); rt.wait_job(j, 60)
        got = {i: gh.read(0, i) for i in st}
        acts = {n: gh.read(0, g.tid(n)) for n in names}
        T = {**{i: a.copy() for i, a in state.items()}, **ds}
        for op in g.ops:
            O.apply_op(op, T, shapes)
        e = {n: rel(acts[n], T[g.tid(n)]) for n in names}
        es = {g.tensors[i].name: rel(got[i], T[i]) for i in st if st[i].dtype == np.float32}
        h1 = T[g.tid("h1")]; z = np.abs(T[g.tid("z1")] + T[g.tid("b1")])
        m = max(list(e.values()) + list(es.values()))
        print(it, f"max {m:.1e}", "near-kink", int((z < 1e-5).sum()), {k: f"{v:.0e}" for k, v in {**e, **es}.items() if v > 1e-5})
        state = got  # continue from the GPU's state
