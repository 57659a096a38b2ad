"""Synthetic workload graphs shaped like the paper's (BASELINE.json ``configs``).

Workload spec only (see sf_inputs/ir.py): these builders say which tensors and ops
a job has; they do not compute anything.

* C1 ``mlp_train``: 2-layer MLP 784-256-10, SGD-momentum, batch 64
  (SURVEY.md section 8(c) op list o1..o11; TF MomentumOptimizer constants, reading Q8).
* C2 ``resnet50_forest``: the exact Keras ResNet-50 variable list (Table 1,
  PAPER.md:1171-1182, lists ResNet50's stateful variables) with per-layer
  softmax-regression compute over the fixed op set (SURVEY.md reading Q16).
* C3 ``bert_chain``: BERT-large's 391 variables with Adam (m, v) and a GEMM chain
  (SURVEY.md reading Q16); mid-graph cut after layer 12's forward.
* inference graphs: batch-1 MLP forwards ("each contained only
  one image (BS=1)").

Phase ids drive the PER_LAYER_PHASE partition (the session
partitions the full graph into subgraphs; granularity reading Q2).
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

from .ir import (ACC, ADAM, BIAS_ACT, BIAS_ACT_BWD, COLSUM, DATASET, F32, FEED, GELU, GEMM,
                 GRAD, I32, INPUT, LABEL, OUTPUT, PARAM, RELU, SCALAR_STATE, SGD_MOM,
                 SLOT, SOFTMAX, SOFTMAX_CE, STEP_INC, TA, TB, ACT, Graph)

SGD_LR = 0.01
SGD_MU = 0.9
ADAM_LR = 1e-4
ADAM_B1 = 0.9
ADAM_B2 = 0.999
ADAM_EPS = 1e-8


# ---------------------------------------------------------------------------------
# C1: MLP training graph (generalised to any widths for tiny test graphs)
# ---------------------------------------------------------------------------------
def mlp_train(widths: Sequence[int] = (784, 256, 10), batch: int = 64, pool: int = 16,
              lr: float = SGD_LR, mu: float = SGD_MU, name: str = "mlp",
              act: str = "relu", host_fed: bool = False) -> Graph:
    """Training graph of an MLP with ReLU (or GELU: ``act="gelu"``) hidden layers and
    softmax-CE loss.  A GELU layer's BIAS_ACT also writes its pre-activation u_i, which
    its BIAS_ACT_BWD reads.  ``host_fed``: x, y come from a host
    input stage (sf_attach_feed) instead of FEED ops over DATASET pools.

    For widths (784, 256, 10) this is exactly SURVEY.md 8(c) step 1 (o1..o11) with
    FEED ops for x, y in front (data cursor = step, reading Q3/Q11) and STEP_INC
    at the end of the update subgraph.  Phases: layer i forward = phase i-1,
    backward of the last layer = phase L, backward of layer i<L = phase 2L-i,
    update = phase 2L.  For L = 2 this gives S0..S4 of SURVEY.md 8(c) step 2.
    """
    L = len(widths) - 1
    g = Graph(name)
    W, b = [], []
    for i in range(L):
        W.append(g.add(f"W{i+1}", widths[i], widths[i + 1], F32, PARAM))
        b.append(g.add(f"b{i+1}", 1, widths[i + 1], F32, PARAM))
    aW, ab = [], []
    for i in range(L):
        aW.append(g.add(f"aW{i+1}", widths[i], widths[i + 1], F32, SLOT))
        ab.append(g.add(f"ab{i+1}", 1, widths[i + 1], F32, SLOT))
    step = g.add("step", 1, 1, I32, SCALAR_STATE)
    if not host_fed:
        xpool = g.add("X_pool", pool * batch, widths[0], F32, DATASET)
        ypool = g.add("Y_pool", pool * batch, 1, I32, DATASET)
    x = g.add("x", batch, widths[0], F32, INPUT)
    y = g.add("y", batch, 1, I32, LABEL)

    # forward
    h_prev = x
    hs: List[int] = []
    us: List[int] = []
    gelu = act == "gelu"
    for i in range(L):
        ph = i
        if i == 0 and not host_fed:
            g.op(FEED, [xpool, step], [x], phase=ph)
            g.op(FEED, [ypool, step], [y], phase=ph)
        z = g.add(f"z{i+1}", batch, widths[i + 1], F32, ACT)
        g.op(GEMM, [h_prev, W[i]], [z], phase=ph)
        last = i == L - 1
        h = g.add("logits" if last else f"h{i+1}", batch, widths[i + 1], F32, ACT)
        if gelu and not last:
            u = g.add(f"u{i+1}", batch, widths[i + 1], F32, ACT)
            g.op(BIAS_ACT, [z, b[i]], [h, u], flags=GELU, phase=ph)
            us.append(u)
        else:
            g.op(BIAS_ACT, [z, b[i]], [h], flags=0 if last else RELU, phase=ph)
            us.append(h)
        hs.append(h)
        h_prev = h
    loss = g.add("loss", 1, 1, F32, OUTPUT)
    dl = g.add("dl", batch, widths[L], F32, GRAD)
    g.op(SOFTMAX_CE, [hs[-1], y], [loss, dl], phase=L - 1)

    # backward
    dW = [None] * L
    db = [None] * L
    d_out = dl  # gradient w.r.t. the pre-activation of layer L (logits = z + b)
    for i in range(L - 1, -1, -1):
        ph = L if i == L - 1 else 2 * L - 1 - i
        inp = x if i == 0 else hs[i - 1]
        if i == L - 1:
            dWi = g.add(f"dW{i+1}", widths[i], widths[i + 1], F32, GRAD)
            g.op(GEMM, [inp, d_out], [dWi], flags=TA, phase=ph)
            dbi = g.add(f"db{i+1}", 1, widths[i + 1], F32, GRAD)
            g.op(COLSUM, [d_out], [dbi], phase=ph)
        else:
            dz = g.add(f"dz{i+1}", batch, widths[i + 1], F32, GRAD)
            dbi = g.add(f"db{i+1}", 1, widths[i + 1], F32, GRAD)
            g.op(BIAS_ACT_BWD, [d_out, us[i]], [dz, dbi], flags=GELU if gelu else 0, phase=ph)
            dWi = g.add(f"dW{i+1}", widths[i], widths[i + 1], F32, GRAD)
            g.op(GEMM, [inp, dz], [dWi], flags=TA, phase=ph)
            d_out = dz
        dW[i], db[i] = dWi, dbi
        if i > 0:
            dh = g.add(f"dh{i}", batch, widths[i], F32, GRAD)
            g.op(GEMM, [d_out, W[i]], [dh], flags=TB, phase=ph)
            d_out = dh
    # update (indivisible subgraph, reading Q2)
    up = 2 * L
    for i in range(L):
        g.op(SGD_MOM, [dW[i]], [W[i], aW[i]], f=[lr, mu], phase=up)
        g.op(SGD_MOM, [db[i]], [b[i], ab[i]], f=[lr, mu], phase=up)
    g.op(STEP_INC, [], [step], phase=up)
    return g


def mlp_infer(widths: Sequence[int] = (784, 256, 10), batch: int = 1,
              name: str = "mlp_infer", wt: bool = False) -> Graph:
    """Batch-1 inference forward: GEMM -> bias+ReLU -> ... -> softmax.

    ``wt``: weights stored output-major, W_i as [N][K] with GEMM flag TB (z = h W_i^T) — the
    serving layout in which every output is a dot product with one contiguous weight row
    (reading Q30)."""
    L = len(widths) - 1
    g = Graph(name)
    W, b = [], []
    for i in range(L):
        shape = (widths[i + 1], widths[i]) if wt else (widths[i], widths[i + 1])
        W.append(g.add(f"W{i+1}", *shape, F32, PARAM))
        b.append(g.add(f"b{i+1}", 1, widths[i + 1], F32, PARAM))
    x = g.add("x", batch, widths[0], F32, INPUT)
    h = x
    for i in range(L):
        z = g.add(f"z{i+1}", batch, widths[i + 1], F32, ACT)
        g.op(GEMM, [h, W[i]], [z], flags=TB if wt else 0)
        last = i == L - 1
        hn = g.add("logits" if last else f"h{i+1}", batch, widths[i + 1], F32, ACT)
        g.op(BIAS_ACT, [z, b[i]], [hn], flags=0 if last else RELU)
        h = hn
    probs = g.add("probs", batch, widths[L], F32, OUTPUT)
    g.op(SOFTMAX, [h], [probs])
    return g


# ---------------------------------------------------------------------------------
# C2: ResNet-50-shaped state (Keras applications variable list)
# ---------------------------------------------------------------------------------
def resnet50_layers() -> List[Tuple[str, int, int, int, int, bool]]:
    """Keras ResNet50 conv/fc layers in creation order.

    Returns (name, k, cin, cout, out_spatial, has_bn).  53 convs (each with bias and a
    BatchNorm with gamma, beta, moving mean, moving var) + fc 2048->1000.
    Parameter count 25,636,712 (Keras applications); Table 1 lists ResNet50 at
    198.53 MiB of stateful variables.
    """
    layers = [("conv1", 7, 3, 64, 112, True)]
    cin = 64
    stages = [(2, 64, 3, 56), (3, 128, 4, 28), (4, 256, 6, 14), (5, 512, 3, 7)]
    for s, f, nblocks, hw in stages:
        for bi in range(1, nblocks + 1):
            pre = f"conv{s}_block{bi}"
            if bi == 1:
                layers.append((pre + "_0", 1, cin, 4 * f, hw, True))
            layers.append((pre + "_1", 1, cin if bi == 1 else 4 * f, f, hw, True))
            layers.append((pre + "_2", 3, f, f, hw, True))
            layers.append((pre + "_3", 1, f, 4 * f, hw, True))
        cin = 4 * f
    layers.append(("fc", 1, 2048, 1000, 1, False))
    return layers


def vgg_layers(depth: int = 16) -> List[Tuple[str, int, int, int, int, bool]]:
    """Keras VGG16 / VGG19 layers (convs with bias, 3 fc); 138,357,544 / 143,667,240 params.

    Used only for the Table 1 identity pin (VGG16 1055.58 MiB and
    VGG19 1096.09 MiB of stateful variables = 2 x params x 4 B, i.e. weights + one
    optimizer slot).
    """
    n3 = 3 if depth == 16 else 4
    cfg = [64, 64, 0, 128, 128, 0] + [256] * n3 + [0] + [512] * n3 + [0] + [512] * n3 + [0]
    layers, cin, hw, i = [], 3, 224, 0
    for c in cfg:
        if c == 0:
            hw //= 2
            continue
        i += 1
        layers.append((f"conv{i}", 3, cin, c, hw, False))
        cin = c
    layers += [("fc1", 1, 25088, 4096, 1, False), ("fc2", 1, 4096, 4096, 1, False),
               ("fc3", 1, 4096, 1000, 1, False)]
    return layers


def forest(layers, batch: int = 8, spatial_div: int = 1, lr: float = SGD_LR,
           mu: float = SGD_MU, name: str = "forest") -> Graph:
    """Per-layer softmax-regression training job over a CNN's variable list (reading Q16).

    Layer l trains logits = X_l W_l + b_l (+ gamma_l + beta_l when it has BN) over Cout
    classes, with X_l a read-only DATASET of shape [M_l, k*k*Cin] where
    M_l = batch * (H_l / spatial_div)^2 (the conv's implicit-GEMM M; fc: M = batch).
    BN moving statistics are passive (migrated, never written).  One phase per
    layer (forward + weight gradient), then the indivisible SGD-momentum update.
    """
    g = Graph(name)
    lay = []
    for (ln, k, cin, cout, hw, bn) in layers:
        K = k * k * cin
        ent = {"name": ln, "K": K, "N": cout, "bn": bn}
        ent["W"] = g.add(ln + "_kernel", K, cout, F32, PARAM)
        ent["b"] = g.add(ln + "_bias", 1, cout, F32, PARAM)
        if bn:
            ent["gamma"] = g.add(ln + "_bn_gamma", 1, cout, F32, PARAM)
            ent["beta"] = g.add(ln + "_bn_beta", 1, cout, F32, PARAM)
            ent["mean"] = g.add(ln + "_bn_moving_mean", 1, cout, F32, PARAM)
            ent["var"] = g.add(ln + "_bn_moving_var", 1, cout, F32, PARAM)
        sp = max(1, hw // spatial_div) if hw > 1 else 1
        ent["M"] = batch * sp * sp
        lay.append(ent)
    for ent in lay:
        ln = ent["name"]
        ent["aW"] = g.add(ln + "_kernel_momentum", ent["K"], ent["N"], F32, SLOT)
        ent["ab"] = g.add(ln + "_bias_momentum", 1, ent["N"], F32, SLOT)
        if ent["bn"]:
            ent["agamma"] = g.add(ln + "_bn_gamma_momentum", 1, ent["N"], F32, SLOT)
            ent["abeta"] = g.add(ln + "_bn_beta_momentum", 1, ent["N"], F32, SLOT)
    step = g.add("step", 1, 1, I32, SCALAR_STATE)
    for ent in lay:
        ent["X"] = g.add(ent["name"] + "_X", ent["M"], ent["K"], F32, DATASET)
        ent["Y"] = g.add(ent["name"] + "_Y", ent["M"], 1, I32, DATASET)
    for li, ent in enumerate(lay):
        ln, M, N = ent["name"], ent["M"], ent["N"]
        z = g.add(ln + "_z", M, N, F32, ACT)
        logits = g.add(ln + "_logits", M, N, F32, ACT)
        loss = g.add(ln + "_loss", 1, 1, F32, OUTPUT)
        dl = g.add(ln + "_dlogits", M, N, F32, GRAD)
        dW = g.add(ln + "_dW", ent["K"], N, F32, GRAD)
        db = g.add(ln + "_db", 1, N, F32, GRAD)
        biases = [ent["b"]] + ([ent["gamma"], ent["beta"]] if ent["bn"] else [])
        g.op(GEMM, [ent["X"], ent["W"]], [z], phase=li)
        g.op(BIAS_ACT, [z] + biases, [logits], flags=0, phase=li)
        g.op(SOFTMAX_CE, [logits, ent["Y"]], [loss, dl], phase=li)
        g.op(GEMM, [ent["X"], dl], [dW], flags=TA, phase=li)
        g.op(COLSUM, [dl], [db], phase=li)
        ent["dW"], ent["db"] = dW, db
    up = len(lay)
    for ent in lay:
        g.op(SGD_MOM, [ent["dW"]], [ent["W"], ent["aW"]], f=[lr, mu], phase=up)
        g.op(SGD_MOM, [ent["db"]], [ent["b"], ent["ab"]], f=[lr, mu], phase=up)
        if ent["bn"]:
            g.op(SGD_MOM, [ent["db"]], [ent["gamma"], ent["agamma"]], f=[lr, mu], phase=up)
            g.op(SGD_MOM, [ent["db"]], [ent["beta"], ent["abeta"]], f=[lr, mu], phase=up)
    g.op(STEP_INC, [], [step], phase=up)
    return g


def resnet50_forest(batch: int = 8, spatial_div: int = 1, lr: float = SGD_LR,
                    mu: float = SGD_MU, max_layers: int | None = None,
                    name: str = "resnet50_forest") -> Graph:
    """C2: the Keras ResNet-50 variable list (534 tensors, 204,881,216 B of params +
    momentum) trained as a per-layer forest (see ``forest``)."""
    layers = resnet50_layers()
    if max_layers is not None:
        layers = layers[:max_layers]
    return forest(layers, batch=batch, spatial_div=spatial_div, lr=lr, mu=mu, name=name)


# ---------------------------------------------------------------------------------
# C3: BERT-large-shaped state with Adam
# ---------------------------------------------------------------------------------
def bert_chain(layers: int = 24, hidden: int = 1024, inter: int = 4096, vocab: int = 30522,
               tokens: int = 512, positions: int = 512, lr: float = ADAM_LR,
               b1: float = ADAM_B1, b2: float = ADAM_B2, eps: float = ADAM_EPS,
               name: str = "bert_chain", act: str = "relu") -> Graph:
    """BERT-large variables (391 tensors, 335,141,888 params at defaults) + Adam.

    ``act="gelu"``: the FFN intermediate Linear uses GELU (where BERT has it; its
    pre-activation is kept for the backward), the other Linears stay ReLU.

    Compute (reading Q16): x0 = pos[:tokens] + embLN_gamma + embLN_beta (requires
    tokens == positions); per layer six Linear+ReLU (q, k, v, o with LN1 gamma/beta as
    extra additive biases on o; intermediate; output with LN2 gamma/beta); pooler;
    head logits = h . word^T; softmax-CE over the vocabulary.  The token-type table is
    passive (never read, never updated).  Phases: one per layer forward (embedding
    in phase 0), pooler+head+loss, one per layer backward, update.
    """
    assert tokens == positions, "x0 is the position table itself (reading Q16)"
    g = Graph(name)
    P = {}
    P["word"] = g.add("word_embeddings", vocab, hidden, F32, PARAM)
    P["pos"] = g.add("position_embeddings", positions, hidden, F32, PARAM)
    P["type"] = g.add("token_type_embeddings", 2, hidden, F32, PARAM)
    P["eg"] = g.add("emb_ln_gamma", 1, hidden, F32, PARAM)
    P["eb"] = g.add("emb_ln_beta", 1, hidden, F32, PARAM)
    lin_names = ["q", "k", "v", "o", "i", "out"]
    dims = {"q": (hidden, hidden), "k": (hidden, hidden), "v": (hidden, hidden),
            "o": (hidden, hidden), "i": (hidden, inter), "out": (inter, hidden)}
    L = []
    for l in range(layers):
        d = {}
        for nm in lin_names:
            kin, kout = dims[nm]
            d["W" + nm] = g.add(f"l{l}_{nm}_kernel", kin, kout, F32, PARAM)
            d["b" + nm] = g.add(f"l{l}_{nm}_bias", 1, kout, F32, PARAM)
            if nm == "o":
                d["g1"] = g.add(f"l{l}_ln1_gamma", 1, hidden, F32, PARAM)
                d["be1"] = g.add(f"l{l}_ln1_beta", 1, hidden, F32, PARAM)
            if nm == "out":
                d["g2"] = g.add(f"l{l}_ln2_gamma", 1, hidden, F32, PARAM)
                d["be2"] = g.add(f"l{l}_ln2_beta", 1, hidden, F32, PARAM)
        L.append(d)
    P["Wp"] = g.add("pooler_kernel", hidden, hidden, F32, PARAM)
    P["bp"] = g.add("pooler_bias", 1, hidden, F32, PARAM)
    params = [i for i, t in enumerate(g.tensors) if t.kind == PARAM]
    mslot = {p: g.add(g.tensors[p].name + "_m", g.tensors[p].rows, g.tensors[p].cols, F32, SLOT)
             for p in params}
    vslot = {p: g.add(g.tensors[p].name + "_v", g.tensors[p].rows, g.tensors[p].cols, F32, SLOT)
             for p in params}
    step = g.add("step", 1, 1, I32, SCALAR_STATE)
    Y = g.add("Y", tokens, 1, I32, DATASET)

    # forward
    x0 = g.add("x0", tokens, hidden, F32, ACT)
    g.op(BIAS_ACT, [P["pos"], P["eg"], P["eb"]], [x0], flags=0, phase=0)
    h = x0
    acts = []  # per layer: list of (input, output, W, biases)
    for l in range(layers):
        rec = []
        for nm in lin_names:
            kin, kout = dims[nm]
            z = g.add(f"l{l}_{nm}_z", tokens, kout, F32, ACT)
            g.op(GEMM, [h, L[l]["W" + nm]], [z], phase=l)
            bs = [L[l]["b" + nm]]
            if nm == "o":
                bs += [L[l]["g1"], L[l]["be1"]]
            if nm == "out":
                bs += [L[l]["g2"], L[l]["be2"]]
            hn = g.add(f"l{l}_{nm}_h", tokens, kout, F32, ACT)
            if act == "gelu" and nm == "i":
                u = g.add(f"l{l}_{nm}_u", tokens, kout, F32, ACT)
                g.op(BIAS_ACT, [z] + bs, [hn, u], flags=GELU, phase=l)
                rec.append((h, u, L[l]["W" + nm], bs, GELU))
            else:
                g.op(BIAS_ACT, [z] + bs, [hn], flags=RELU, phase=l)
                rec.append((h, hn, L[l]["W" + nm], bs, 0))
            h = hn
        acts.append(rec)
    ph = layers
    zp = g.add("pool_z", tokens, hidden, F32, ACT)
    g.op(GEMM, [h, P["Wp"]], [zp], phase=ph)
    hp = g.add("pool_h", tokens, hidden, F32, ACT)
    g.op(BIAS_ACT, [zp, P["bp"]], [hp], flags=RELU, phase=ph)
    logits = g.add("logits", tokens, vocab, F32, ACT)
    g.op(GEMM, [hp, P["word"]], [logits], flags=TB, phase=ph)
    loss = g.add("loss", 1, 1, F32, OUTPUT)
    dl = g.add("dlogits", tokens, vocab, F32, GRAD)
    g.op(SOFTMAX_CE, [logits, Y], [loss, dl], phase=ph)
    # backward: head + pooler (phase layers+1)
    ph = layers + 1
    grads = {}
    gword = g.add("word_embeddings_grad", vocab, hidden, F32, GRAD)
    g.op(GEMM, [dl, hp], [gword], flags=TA, phase=ph)
    grads[P["word"]] = gword
    dhp = g.add("pool_dh", tokens, hidden, F32, GRAD)
    g.op(GEMM, [dl, P["word"]], [dhp], phase=ph)
    dzp = g.add("pool_dz", tokens, hidden, F32, GRAD)
    gbp = g.add("pooler_bias_grad", 1, hidden, F32, GRAD)
    g.op(BIAS_ACT_BWD, [dhp, hp], [dzp, gbp], phase=ph)
    grads[P["bp"]] = gbp
    gWp = g.add("pooler_kernel_grad", hidden, hidden, F32, GRAD)
    g.op(GEMM, [h, dzp], [gWp], flags=TA, phase=ph)
    grads[P["Wp"]] = gWp
    dh = g.add("pool_dx", tokens, hidden, F32, GRAD)
    g.op(GEMM, [dzp, P["Wp"]], [dh], flags=TB, phase=ph)
    for l in range(layers - 1, -1, -1):
        ph = layers + 2 + (layers - 1 - l)
        for j in range(len(lin_names) - 1, -1, -1):
            nm = lin_names[j]
            inp, out, Wt, bs, fl = acts[l][j]
            kin, kout = dims[nm]
            dz = g.add(f"l{l}_{nm}_dz", tokens, kout, F32, GRAD)
            gb = g.add(f"l{l}_{nm}_bias_grad", 1, kout, F32, GRAD)
            g.op(BIAS_ACT_BWD, [dh, out], [dz, gb], flags=fl, phase=ph)
            for bt in bs:
                grads[bt] = gb  # additive biases share the column-sum gradient
            gW = g.add(f"l{l}_{nm}_kernel_grad", kin, kout, F32, GRAD)
            g.op(GEMM, [inp, dz], [gW], flags=TA, phase=ph)
            grads[Wt] = gW
            dx = g.add(f"l{l}_{nm}_dx", tokens, kin, F32, GRAD)
            g.op(GEMM, [dz, Wt], [dx], flags=TB, phase=ph)
            dh = dx
    # embedding: x0 = pos + eg + eb  =>  dpos = dx0, deg = deb = colsum(dx0)
    ph = 2 * layers + 2
    grads[P["pos"]] = dh
    gemb = g.add("emb_ln_grad", 1, hidden, F32, GRAD)
    g.op(COLSUM, [dh], [gemb], phase=ph - 1)
    grads[P["eg"]] = gemb
    grads[P["eb"]] = gemb
    for p in params:
        if p == P["type"]:
            continue  # passive token-type table
        g.op(ADAM, [grads[p], step], [p, mslot[p], vslot[p]], f=[lr, b1, b2, eps], phase=ph)
    g.op(STEP_INC, [], [step], phase=ph)
    return g


def bert_mid_cut_phase(layers: int = 24, after_layer: int = 12) -> int:
    """Cut index of the boundary right after layer ``after_layer``'s forward (C3)."""
    return after_layer
