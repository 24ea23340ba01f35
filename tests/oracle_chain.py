"""Oracle composition of a whole split stack (region + unsplit tail), for the stack parity test.
Composes oracle.ops only.  ``round_bf16`` emulates the bf16 STORAGE of every activation and
gradient level (the exact inputs the bf16 GPU path feeds each op); arithmetic stays
fp64."""
from __future__ import annotations

import numpy as np

import synth
from oracle import ops as O
from oracle import plan as OP


def _rnd(P, on):
    if not on:
        return P
    return [[synth.to_bf16_f32(p.astype(np.float32)).astype(np.float64) for p in row] for row in P]


def _masked(layers, m, prev_masked):
    if m == 0:
        return prev_masked
    l = layers[m - 1]
    return l["op"] == "conv" and l.get("relu", True)


def run(region, tail, N, C, H, W, Oh, Ow, params, X, G, round_bf16=False):
    """Returns (output NCHW, [dW OIHW per conv in order], [db per conv], pools) where pools maps
    (key, m) -> (pool input patches, argmax patches) for the argmax-agreement check."""
    rp = OP.plan(region, N, C, H, W, Oh, Ow)
    Lr = rp.layers[-1]
    tp = OP.plan(tail, N, region[-1]["cout"], Lr.H_out, Lr.W_out,
                 [0, _out(tail, Lr.H_out, 0)], [0, _out(tail, Lr.W_out, 1)]) if tail else None
    pit = iter(params)
    prm = {}
    for key, layers in (("r", region), ("t", tail)):
        for m, l in enumerate(layers):
            if l["op"] == "conv":
                prm[(key, m)] = next(pit)

    def fwd(key, plan, layers, P):
        acts, args = [P], {}
        for m, (l, lp) in enumerate(zip(layers, plan.layers)):
            if l["op"] == "conv":
                Wt, b = prm[(key, m)]
                P = O.conv_fwd(P, Wt, b, lp, l.get("relu", True))
            else:
                P, args[m] = O.pool_fwd(P, lp)
            P = _rnd(P, round_bf16)
            acts.append(P)
        return acts, args

    def bwd(key, plan, layers, acts, args, g, first_masked, need_input):
        grads = {}
        for m in range(len(layers) - 1, -1, -1):
            l, lp = layers[m], plan.layers[m]
            msk = _masked(layers, m, first_masked)
            last = m == 0 and not need_input
            if l["op"] == "conv":
                Wt, _ = prm[(key, m)]
                grads[m] = O.conv_bwd_filter(acts[m], g, lp)
                if not last:
                    g = _rnd(O.conv_bwd_data(g, Wt, lp, acts[m] if msk else None), round_bf16)
            else:
                g = O.pool_bwd(g, args[m], lp)
                if msk:
                    g = O.relu_mask(g, acts[m])
                g = _rnd(g, round_bf16)
        return g, grads

    def top_mask(layers, acts, g):
        """loss = <Y, G> with Y the stack OUTPUT: when the last op is a conv with a
        fused ReLU, G reaches the conv's pre-activation only where Y > 0."""
        l = layers[-1]
        return O.relu_mask(g, acts[-1]) if l["op"] == "conv" and l.get("relu", True) else g

    pools = {}
    acts_r, args_r = fwd("r", rp, region, _rnd(O.split(X, rp.layers[0].Ih, rp.layers[0].Iw), round_bf16))
    out = O.merge(acts_r[-1])
    pools.update({("r", m): (acts_r[m], a) for m, a in args_r.items()})
    region_out_masked = _masked(region, len(region), False)
    if tp is not None:
        acts_t, args_t = fwd("t", tp, tail, [[out]])
        pools.update({("t", m): (acts_t[m], a) for m, a in args_t.items()})
        out = O.merge(acts_t[-1])
        g, grads_t = bwd("t", tp, tail, acts_t, args_t, top_mask(tail, acts_t, [[G]]), region_out_masked, True)
        g = O.split(O.merge(g), Lr.Oh, Lr.Ow)
    else:
        g, grads_t = top_mask(region, acts_r, O.split(G, Lr.Oh, Lr.Ow)), {}
    _, grads_r = bwd("r", rp, region, acts_r, args_r, g, False, False)
    dWs, dbs = [], []
    for key, layers, grads in (("r", region, grads_r), ("t", tail, grads_t)):
        for m, l in enumerate(layers):
            if l["op"] == "conv":
                dWs.append(grads[m][0])
                dbs.append(grads[m][1])
    return out, dWs, dbs, pools


def _out(layers, L, dim):
    for l in layers:
        k, s = (l["kh"], l["sh"]) if dim == 0 else (l["kw"], l["sw"])
        pb, pe = (l["ph_b"], l["ph_e"]) if dim == 0 else (l["pw_b"], l["pw_e"])
        L = (L + pb + pe - k) // s + 1
    return L


def run_resnet(chain, blocks, N, C, H, W, Oh, Ow, params, X, G, round_bf16=False, return_input_grad=False):
    """Oracle composition of the BN-free ResNet split stack (synth.resnet18_blocks): the main
    chain with a residual join after every block's second conv, the 1x1 downsample on its own
    one-layer plan sharing the block's output partition.  G is the gradient of the merged output.
    Returns (output NCHW, dWs, dbs) with dWs/dbs in synth.resnet_params order (chain convs, then
    downsample convs)."""
    rp = OP.plan(chain, N, C, H, W, Oh, Ow)
    nconv = sum(1 for l in chain if l["op"] == "conv")
    pit = iter(params)
    prm = {m: next(pit) for m, l in enumerate(chain) if l["op"] == "conv"}
    ds = {}
    for k, b in enumerate(blocks):
        if b["ds"] is not None:
            lo = rp.layers[b["a"] + 1]
            li = rp.layers[b["a"]]
            dp = OP.plan([b["ds"]], N, b["ds"]["cin"], li.H_in, li.W_in, lo.Oh, lo.Ow).layers[0]
            assert dp.Ih == li.Ih and dp.Iw == li.Iw
            ds[k] = (dp, next(pit))
    at = {b["a"]: k for k, b in enumerate(blocks)}
    block_out = {b["a"] + 2 for b in blocks}
    rnd = lambda P: _rnd(P, round_bf16)
    # forward
    acts = [rnd(O.split(X, rp.layers[0].Ih, rp.layers[0].Iw))]
    args, sc_out = {}, {}
    m = 0
    while m < len(chain):
        l, lp = chain[m], rp.layers[m]
        if m in at:
            k = at[m]
            Wa, ba = prm[m]
            Wb, bb = prm[m + 1]
            h = rnd(O.conv_fwd(acts[m], Wa, ba, lp, True))
            # the block output y = ReLU(conv_b(h) + s) is the stored level; conv_b's own output is never stored
            # (the join is fused into its epilogue), so only y is rounded to the storage type (R13)
            z = O.conv_fwd(h, Wb, bb, rp.layers[m + 1], False)
            if k in ds:
                dp, (Wd, bd) = ds[k]
                s = sc_out[k] = rnd(O.conv_fwd(acts[m], Wd, bd, dp, False))
            else:
                s = acts[m]
            acts += [h, rnd(O.residual_add(z, s, relu=True))]
            m += 2
            continue
        if l["op"] == "conv":
            Wt, b = prm[m]
            acts.append(rnd(O.conv_fwd(acts[m], Wt, b, lp, l.get("relu", True))))
        else:
            P, args[m] = O.pool_fwd(acts[m], lp)
            acts.append(rnd(P))
        m += 1
    out = O.merge(acts[-1])
    # backward
    grads, gds = {}, {}
    g = rnd(O.relu_mask(O.split(G, rp.layers[-1].Oh, rp.layers[-1].Ow), acts[-1]))
    m = len(chain) - 1
    while m >= 0:
        a = m - 1
        if a in at:
            k = at[a]
            Wa, _ = prm[a]
            Wb, _ = prm[a + 1]
            grads[a + 1] = O.conv_bwd_filter(acts[a + 1], g, rp.layers[a + 1])
            gh = rnd(O.conv_bwd_data(g, Wb, rp.layers[a + 1], acts[a + 1]))
            grads[a] = O.conv_bwd_filter(acts[a], gh, rp.layers[a])
            gx = rnd(O.conv_bwd_data(gh, Wa, rp.layers[a]))
            if k in ds:
                dp, (Wd, _) = ds[k]
                gds[k] = O.conv_bwd_filter(acts[a], g, dp)
                gs = rnd(O.conv_bwd_data(g, Wd, dp))
            else:
                gs = g
            gsum = O.residual_add(gx, gs)
            g = rnd(O.relu_mask(gsum, acts[a]) if a in block_out else gsum)
            m = a - 1
            continue
        l, lp = chain[m], rp.layers[m]
        if l["op"] == "conv":
            grads[m] = O.conv_bwd_filter(acts[m], g, lp)
            if m > 0:
                g = rnd(O.conv_bwd_data(g, prm[m][0], lp, acts[m] if _masked(chain, m, False) else None))
        else:
            g = O.pool_bwd(g, args[m], lp)
            if _masked(chain, m, False):
                g = O.relu_mask(g, acts[m])
            g = rnd(g)
        m -= 1
    dWs = [grads[m][0] for m in sorted(grads)] + [gds[k][0] for k in sorted(gds)]
    dbs = [grads[m][1] for m in sorted(grads)] + [gds[k][1] for k in sorted(gds)]
    assert len(dWs) == nconv + len(ds)
    if return_input_grad:
        return out, dWs, dbs, O.merge(g)
    return out, dWs, dbs


def run_resnet_bn(chain, blocks, N, C, H, W, Oh, Ow, params, bn, X, G, round_bf16=False, eps=1e-5):
    """Oracle composition of the ResNet split stack WITH whole-tensor BN (R11): conv (no bias) -> BN
    -> ReLU; y = ReLU(BN_b(conv_b(h)) + shortcut), shortcut = x | BN_ds(ds(x)).  ``params`` = (W, _)
    per conv (biases unused), ``bn`` = (gamma, beta) per conv, both in synth.resnet_params order.
    Returns (output NCHW, dWs, dgammas, dbetas)."""
    rp = OP.plan(chain, N, C, H, W, Oh, Ow)
    conv_ms = [m for m, l in enumerate(chain) if l["op"] == "conv"]
    prm = {m: params[i][0] for i, m in enumerate(conv_ms)}
    bnp = {("r", m): bn[i] for i, m in enumerate(conv_ms)}
    ds, i = {}, len(conv_ms)
    for k, b in enumerate(blocks):
        if b["ds"] is not None:
            lo, li = rp.layers[b["a"] + 1], rp.layers[b["a"]]
            dp = OP.plan([b["ds"]], N, b["ds"]["cin"], li.H_in, li.W_in, lo.Oh, lo.Ow).layers[0]
            ds[k] = (dp, params[i][0])
            bnp[("ds", k)] = bn[i]
            i += 1
    at = {b["a"]: k for k, b in enumerate(blocks)}
    block_out = {b["a"] + 2 for b in blocks}
    rnd = lambda P: _rnd(P, round_bf16)
    zero = lambda Wt: np.zeros(Wt.shape[0])
    st = {}   # key -> (z, y, mean, invstd, relu)

    def cbn(key, Xp, Wt, lp, relu):
        z = rnd(O.conv_fwd(Xp, Wt, zero(Wt), lp, False))
        y, mean, inv = O.batch_norm(z, *bnp[key], eps=eps, relu=relu)
        y = rnd(y)
        st[key] = (z, y, mean, inv, relu)
        return y

    inp = {0: rnd(O.split(X, rp.layers[0].Ih, rp.layers[0].Iw))}
    args = {}
    m = 0
    while m < len(chain):
        l, lp = chain[m], rp.layers[m]
        if m in at:
            k = at[m]
            h = cbn(("r", m), inp[m], prm[m], lp, True)
            inp[m + 1] = h
            zb = cbn(("r", m + 1), h, prm[m + 1], rp.layers[m + 1], False)
            s = cbn(("ds", k), inp[m], ds[k][1], ds[k][0], False) if k in ds else inp[m]
            inp[m + 2] = rnd(O.residual_add(zb, s, relu=True))
            m += 2
            continue
        if l["op"] == "conv":
            inp[m + 1] = cbn(("r", m), inp[m], prm[m], lp, True)
        else:
            P, args[m] = O.pool_fwd(inp[m], lp)
            inp[m + 1] = rnd(P)
        m += 1
    nl = len(chain)
    out = O.merge(inp[nl])
    grads, bgrads = {}, {}

    def bn_bwd(key, g):
        z, y, mean, inv, relu = st[key]
        dz, dgm, dbt = O.batch_norm_bwd(g, z, y, bnp[key][0], mean, inv, relu=False)
        bgrads[key] = (dgm, dbt)
        return rnd(dz)

    g = rnd(O.relu_mask(O.split(G, rp.layers[-1].Oh, rp.layers[-1].Ow), inp[nl]))
    m = nl - 1
    while m >= 0:
        a = m - 1
        if a in at:
            k = at[a]
            gzb = bn_bwd(("r", a + 1), g)
            grads[("r", a + 1)] = O.conv_bwd_filter(inp[a + 1], gzb, rp.layers[a + 1])[0]
            gh = O.conv_bwd_data(gzb, prm[a + 1], rp.layers[a + 1])
            gh = rnd(O.relu_mask(gh, inp[a + 1]))               # ReLU of BN_a (applied inside BN bwd on the GPU)
            gza = bn_bwd(("r", a), gh)
            grads[("r", a)] = O.conv_bwd_filter(inp[a], gza, rp.layers[a])[0]
            gx = rnd(O.conv_bwd_data(gza, prm[a], rp.layers[a]))
            if k in ds:
                dp, Wd = ds[k]
                gzd = bn_bwd(("ds", k), g)
                grads[("ds", k)] = O.conv_bwd_filter(inp[a], gzd, dp)[0]
                gs = rnd(O.conv_bwd_data(gzd, Wd, dp))
            else:
                gs = g
            gsum = O.residual_add(gx, gs)
            g = rnd(O.relu_mask(gsum, inp[a]) if a in block_out else gsum)
            m = a - 1
            continue
        l, lp = chain[m], rp.layers[m]
        if l["op"] == "conv":
            gz = bn_bwd(("r", m), g)
            grads[("r", m)] = O.conv_bwd_filter(inp[m], gz, lp)[0]
        else:
            g = O.pool_bwd(g, args[m], lp)
            g = rnd(O.relu_mask(g, inp[m]))                     # the stem's BN+ReLU output feeds the pool
        m -= 1
    keys = [("r", m) for m in conv_ms] + [("ds", k) for k in sorted(ds)]
    return out, [grads[k] for k in keys], [bgrads[k][0] for k in keys], [bgrads[k][1] for k in keys]


def run_resnet18_full(rc, rb, tc, tb, N, C, H, W, Oh, Ow, params, X, G, round_bf16=False):
    """Oracle of the whole trunk: split region (stem .. layer2) -> merge -> unsplit tail (layer3,
    layer4; 1x1 split) -> global average pool; G is the gradient of the pooled [N][C] output.
    params in synth.resnet_params order for the region, then for the tail.
    Returns (pooled [N][C], dWs, dbs) in that order."""
    n_r = sum(1 for l in rc if l["op"] == "conv") + sum(1 for b in rb if b["ds"] is not None)
    p_r, p_t = params[:n_r], params[n_r:]
    rp = OP.plan(rc, N, C, H, W, Oh, Ow)
    Lr = rp.layers[-1]
    zero = np.zeros((N, rc[-1]["cout"], Lr.H_out, Lr.W_out))
    out_r, _, _ = run_resnet(rc, rb, N, C, H, W, Oh, Ow, p_r, X, zero, round_bf16)
    tp = OP.plan(tc, N, rc[-1]["cout"], Lr.H_out, Lr.W_out, [0, _out(tc, Lr.H_out, 0)], [0, _out(tc, Lr.W_out, 1)])
    Lt = tp.layers[-1]
    G_t = O.global_avg_pool_bwd(G, Lt.H_out, Lt.W_out)
    if round_bf16:
        G_t = synth.to_bf16_f32(G_t.astype(np.float32)).astype(np.float64)
    out_t, dW_t, db_t, g_in = run_resnet(tc, tb, N, rc[-1]["cout"], Lr.H_out, Lr.W_out, [0, Lt.H_out], [0, Lt.W_out],
                                         p_t, out_r, G_t, round_bf16, return_input_grad=True)
    pooled = O.global_avg_pool(out_t)
    _, dW_r, db_r = run_resnet(rc, rb, N, C, H, W, Oh, Ow, p_r, X, g_in, round_bf16)
    return pooled, dW_r + dW_t, db_r + db_t
