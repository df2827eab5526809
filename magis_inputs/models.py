"""Synthetic training graphs shaped like the paper's workloads (Table 2,
P:1751-1760) -- INPUT GENERATION ONLY.  Sizes come from real shapes and
dtypes; costs from graph.op_cost.  See DESIGN.md §Inputs for the recipes.
"""
from __future__ import annotations

import numpy as np

from .graph import AG, Builder, T, numel


# --------------------------------------------------------------------------
# C1: 10-op diamond (Fig. 2-style toy)
# --------------------------------------------------------------------------

def diamond(branches, seed: int = 1):
    """source -> chains (lengths ``branches``, each >= 2) -> sink.
    Sizes 512 B x U[1, 2^20) (SURVEY §8d C1 recipe), zero costs except 1e-6."""
    rng = np.random.default_rng(seed)
    b = Builder(f"diamond{''.join(map(str, branches))}")
    n = 2 + sum(branches)
    sizes = [512 * int(x) for x in rng.integers(1, 1 << 20, n)]
    src = b.node("src", sizes[0], (), flops=1e3)
    ends = []
    k = 1
    for L in branches:
        prev = src
        for _ in range(L):
            prev = b.node(f"m{k}", sizes[k], [prev], flops=1e3)
            k += 1
        ends.append(prev)
    sink = b.node("sink", sizes[k], ends, flops=1e3)
    b.outputs.add(sink)
    return b.finish()


# --------------------------------------------------------------------------
# C2: ResNet-50 training, b64, 224^2, fp32 (Table 2)
# --------------------------------------------------------------------------

def _bn(ag: AG, name: str, x: T, C: int, stat_shape=None) -> T:
    """BatchNorm as 4 primitives: mean, var, normalize, affine.
    With ``stat_shape`` the statistics have that shape (LayerNorm: one mean /
    variance per token, affine over the last dim C)."""
    g = ag.param(name + ".gamma", (C,))
    bt = ag.param(name + ".beta", (C,))
    N = numel(x.shape)
    sshape = (C,) if stat_shape is None else tuple(stat_shape)

    def mean_bwd(ag_, dy, out, ins):
        x_, = ins
        return [(x_, ag_._g(name + ".mean.d", [dy], x_, N))]
    mu = ag.op(name + ".mean", [x], sshape, N, mean_bwd)

    def var_bwd(ag_, dy, out, ins):
        x_, m_ = ins
        return [(x_, ag_._g(name + ".var.dx", [dy, x_, m_], x_, 3 * N)),
                (m_, ag_._g(name + ".var.dm", [dy, x_, m_], m_, 2 * N))]
    var = ag.op(name + ".var", [x, mu], sshape, 3 * N, var_bwd)

    def norm_bwd(ag_, dy, out, ins):
        x_, m_, v_ = ins
        return [(x_, ag_._g(name + ".norm.dx", [dy, v_], x_, 2 * N)),
                (m_, ag_._g(name + ".norm.dm", [dy, v_], m_, N)),
                (v_, ag_._g(name + ".norm.dv", [dy, x_, m_, v_], v_, 3 * N))]
    nrm = ag.op(name + ".norm", [x, mu, var], x.shape, 3 * N, norm_bwd)

    def aff_bwd(ag_, dy, out, ins):
        n_, g_, b_ = ins
        return [(n_, ag_._g(name + ".aff.dn", [dy, g_], n_, N)),
                (g_, ag_._g(name + ".aff.dg", [dy, n_], g_, 2 * N)),
                (b_, ag_._g(name + ".aff.db", [dy], b_, N))]
    return ag.op(name + ".affine", [nrm, g, bt], x.shape, 2 * N, aff_bwd)


def resnet50(batch: int = 64, img: int = 224, dtype_bytes: int = 4):
    b = Builder(f"resnet50_b{batch}")
    ag = AG(b, dtype_bytes)
    x = ag.input("input", (batch, 3, img, img))

    def conv(name, x, cout, k, stride):
        cin = x.shape[1]
        h = (x.shape[2] + stride - 1) // stride
        w = ag.param(name + ".w", (cout, cin, k, k))
        return ag.conv(name, x, w, (x.shape[0], cout, h, h))

    y = conv("stem.conv", x, 64, 7, 2)
    y = _bn(ag, "stem.bn", y, 64)
    y = ag.unary("stem.relu", y, save="y")
    y = ag.unary("stem.maxpool", y, save="x", shape=(batch, 64, img // 4, img // 4))
    cin = 64
    for si, (nblk, width) in enumerate(zip([3, 4, 6, 3], [64, 128, 256, 512])):
        for bi in range(nblk):
            stride = 2 if (bi == 0 and si > 0) else 1
            p = f"l{si + 1}.{bi}"
            idn = y
            h = conv(p + ".conv1", y, width, 1, 1)
            h = _bn(ag, p + ".bn1", h, width)
            h = ag.unary(p + ".relu1", h, save="y")
            h = conv(p + ".conv2", h, width, 3, stride)
            h = _bn(ag, p + ".bn2", h, width)
            h = ag.unary(p + ".relu2", h, save="y")
            h = conv(p + ".conv3", h, width * 4, 1, 1)
            h = _bn(ag, p + ".bn3", h, width * 4)
            if bi == 0:
                idn = conv(p + ".down.conv", y, width * 4, 1, stride)
                idn = _bn(ag, p + ".down.bn", idn, width * 4)
            h = ag.add(p + ".add", h, idn)
            y = ag.unary(p + ".relu3", h, save="y")
            cin = width * 4
    y = ag.unary("avgpool", y, save="none", shape=(batch, cin))
    wfc = ag.param("fc.w", (cin, 1000))
    bfc = ag.param("fc.b", (1000,))
    lg = ag.matmul("fc", y, wfc, (batch, 1000))
    lg = ag.bias("fc.bias", lg, bfc)
    lab = ag.input("labels", (batch,), kind="label", dbytes=8)
    loss = ag.loss("loss", lg, lab)
    ag.backward(loss)
    return b


# --------------------------------------------------------------------------
# Transformer layers (C3 BERT-large, C5 GPT-Neo-1.3B shape)
# --------------------------------------------------------------------------

def _attention_core(ag: AG, p: str, qkv: T, mask: T, B: int, S: int, H: int, D: int,
                    tag: str | None) -> T:
    """QK^T, scale, mask-add, softmax, dropout, PV -- the F-Trans set S."""
    ag.tag = tag
    dh = D // H
    sc = ag.bmm(p + ".qk", qkv, qkv, (B, H, S, S), 2.0 * B * H * S * S * dh)
    sc = ag.unary(p + ".scale", sc, save="none")
    sc = ag.const_op(p + ".mask", sc, mask, save="none")
    pr = ag.unary(p + ".softmax", sc, save="y", flops_per=5.0)
    pr = ag.unary(p + ".attn_drop", pr, save="y")
    ctx = ag.bmm(p + ".pv", pr, qkv, (B, S, D), 2.0 * B * H * S * S * dh)
    ag.tag = None
    return ctx


def _ffn(ag: AG, p: str, x: T, D: int, Fd: int, tag: str | None) -> T:
    B, S = x.shape[0], x.shape[1]
    w1 = ag.param(p + ".w1", (D, Fd))
    b1 = ag.param(p + ".b1", (Fd,))
    w2 = ag.param(p + ".w2", (Fd, D))
    b2 = ag.param(p + ".b2", (D,))
    ag.tag = tag
    h = ag.matmul(p + ".fc1", x, w1, (B, S, Fd))
    h = ag.bias(p + ".fc1.bias", h, b1)
    h = ag.unary(p + ".gelu", h, save="x", flops_per=8.0)
    h = ag.matmul(p + ".fc2", h, w2, (B, S, D))
    h = ag.bias(p + ".fc2.bias", h, b2)
    ag.tag = None
    return h


def _ln(ag: AG, p: str, x: T, D: int, prims: bool = False) -> T:
    """LayerNorm: one fused op, or (``prims``) 4 primitives like BN with
    per-token statistics."""
    if prims:
        return _bn(ag, p, x, D, stat_shape=x.shape[:-1])
    return ag.norm(p, x, ag.param(p + ".g", (D,)), ag.param(p + ".b", (D,)))


def transformer(name: str, layers: int, D: int, H: int, Fd: int, vocab: int, B: int, S: int,
                dtype_bytes: int, pre_ln: bool, ftrans: int = 1, ln_prims: bool = False):
    """BERT-style (post-LN) or GPT-style (pre-LN) training graph.  With
    ftrans > 1 the attention core and the FFN sub-graph of every layer are
    tagged as F-Trans sets (split along the batch dim) for ftrans.apply."""
    b = Builder(name)
    ag = AG(b, dtype_bytes)
    ids = ag.input("ids", (B, S), dbytes=8)
    wte = ag.param("wte", (vocab, D))
    x = ag.op("embed", [ids, wte], (B, S, D), B * S * D,
              lambda ag_, dy, out, ins: [(ins[1], ag_._g("embed.dW", [dy, ins[0]], ins[1], B * S * D))])
    wpe = ag.param("wpe", (S, D))
    x = ag.add("embed.pos", x, wpe)
    if not pre_ln:
        x = _ln(ag, "embed.ln", x, D)
    x = ag.unary("embed.drop", x, save="y")
    mask = ag.input("mask", (B, 1, 1, S), dbytes=dtype_bytes)
    for li in range(layers):
        p = f"h{li}"
        tag_a = f"{p}.attn" if ftrans > 1 else None
        tag_f = f"{p}.ffn" if ftrans > 1 else None
        res = x
        h = _ln(ag, p + ".ln1", x, D, ln_prims) if pre_ln else x
        wqkv = ag.param(p + ".wqkv", (D, 3 * D))
        bqkv = ag.param(p + ".bqkv", (3 * D,))
        wo = ag.param(p + ".wo", (D, D))
        bo = ag.param(p + ".bo", (D,))
        # the whole attention block (projections + core) is the F-Trans set
        ag.tag = tag_a
        qkv = ag.matmul(p + ".qkv", h, wqkv, (B, S, 3 * D))
        qkv = ag.bias(p + ".qkv.bias", qkv, bqkv)
        ctx = _attention_core(ag, p, qkv, mask, B, S, H, D, tag_a)
        ag.tag = tag_a
        a = ag.matmul(p + ".proj", ctx, wo, (B, S, D))
        a = ag.bias(p + ".proj.bias", a, bo)
        a = ag.unary(p + ".drop1", a, save="y")
        ag.tag = None
        x = ag.add(p + ".res1", a, res)
        if not pre_ln:
            x = _ln(ag, p + ".ln1", x, D)
        res = x
        h = _ln(ag, p + ".ln2", x, D, ln_prims) if pre_ln else x
        f = _ffn(ag, p + ".ffn", h, D, Fd, tag_f)
        ag.tag = tag_f
        f = ag.unary(p + ".drop2", f, save="y")
        ag.tag = None
        x = ag.add(p + ".res2", f, res)
        if not pre_ln:
            x = _ln(ag, p + ".ln2", x, D)
    if pre_ln:
        x = _ln(ag, "ln_f", x, D, ln_prims)
    else:
        wt = ag.param("mlm.w", (D, D))
        x = ag.matmul("mlm.dense", x, wt, (B, S, D))
        x = ag.unary("mlm.gelu", x, save="x", flops_per=8.0)
        x = _ln(ag, "mlm.ln", x, D)
    lg = ag.matmul("lm_head", x, wte, (B, S, vocab))
    lab = ag.input("labels", (B, S), kind="label", dbytes=8)
    loss = ag.loss("loss", lg, lab)
    ag.backward(loss)
    return b


def bert_large(B: int = 32, S: int = 512, ftrans: int = 4, layers: int = 24):
    return transformer(f"bert_large_s{S}_b{B}_ft{ftrans}" + (f"_l{layers}" if layers != 24 else ""), layers,
                       1024, 16, 4096, 30522, B, S, 4, pre_ln=False, ftrans=ftrans)


def gpt_neo_1p3b(B: int = 32, S: int = 512, layers: int = 24):
    """GPT-Neo-1.3B shape; LayerNorm as 4 primitives (SURVEY §8 config sheet:
    ~2.3-2.6k ops, n_total ~3k with R = 128)."""
    return transformer(f"gpt_neo_1.3b_s{S}_b{B}", layers, 2048, 16, 8192, 50257, B, S, 2,
                       pre_ln=True, ftrans=1, ln_prims=True)


# --------------------------------------------------------------------------
# C4: SD-v1-shaped UNet, bf16, batch 8, latent 128x128
# --------------------------------------------------------------------------

def _gn(ag: AG, p: str, x: T, C: int) -> T:
    """GroupNorm as 4 primitives (as BN above)."""
    return _bn(ag, p, x, C)


def unet_sd(B: int = 8, latent: int = 128, chans=(320, 640, 1280, 1280), ctx_len: int = 77,
            ctx_dim: int = 768, heads: int = 8, ftrans: int = 32, down_blocks: int = 2,
            up_blocks: int = 3):
    b = Builder(f"unet_sd_b{B}_{latent * 8}px_ft{ftrans}")
    ag = AG(b, 2)
    x = ag.input("latent", (B, 4, latent, latent))
    temb_in = ag.input("temb", (B, 1280))
    ctx = ag.input("context", (B, ctx_len, ctx_dim))
    attn_id = [0]

    def conv(name, x, cout, k, stride=1):
        h = x.shape[2] // stride
        w = ag.param(name + ".w", (cout, x.shape[1], k, k))
        return ag.conv(name, x, w, (x.shape[0], cout, h, h))

    def resblock(p, x, cout):
        cin = x.shape[1]
        h = _gn(ag, p + ".gn1", x, cin)
        h = ag.unary(p + ".silu1", h, save="x", flops_per=4.0)
        h = conv(p + ".conv1", h, cout, 3)
        wt = ag.param(p + ".temb.w", (1280, cout))
        te = ag.matmul(p + ".temb", temb_in, wt, (B, cout))
        h = ag.add(p + ".temb.add", h, te)
        h = _gn(ag, p + ".gn2", h, cout)
        h = ag.unary(p + ".silu2", h, save="x", flops_per=4.0)
        h = ag.unary(p + ".drop", h, save="y")
        h = conv(p + ".conv2", h, cout, 3)
        if cin != cout:
            x = conv(p + ".skip", x, cout, 1)
        return ag.add(p + ".add", h, x)

    def attn(p, hseq, kv_src, C, cross):
        """q from hseq, k/v from kv_src; core is an F-Trans set split along
        the query-token dim (K, V shared; dK, dV are reduce merges)."""
        Bq, L, _ = hseq.shape
        Lk = kv_src.shape[1]
        dk = kv_src.shape[2]
        wq = ag.param(p + ".wq", (C, C))
        wk = ag.param(p + ".wk", (dk, C))
        wv = ag.param(p + ".wv", (dk, C))
        k = ag.matmul(p + ".k", kv_src, wk, (Bq, Lk, C))
        v = ag.matmul(p + ".v", kv_src, wv, (Bq, Lk, C))
        tag = f"attn{attn_id[0]}" if ftrans > 1 else None
        attn_id[0] += 1
        wo = ag.param(p + ".wo", (C, C))
        ag.tag = tag
        q = ag.matmul(p + ".q", hseq, wq, (Bq, L, C))
        sc = ag.bmm(p + ".qk", q, k, (Bq, heads, L, Lk), 2.0 * Bq * L * Lk * C, b_shared=True)
        sc = ag.unary(p + ".scale", sc, save="none")
        pr = ag.unary(p + ".softmax", sc, save="y", flops_per=5.0)
        o = ag.bmm(p + ".pv", pr, v, (Bq, L, C), 2.0 * Bq * L * Lk * C, b_shared=True)
        o = ag.matmul(p + ".o", o, wo, (Bq, L, C))
        ag.tag = None
        return o

    def transformer_block(p, x):
        Bx, C, Hh, Ww = x.shape
        L = Hh * Ww
        h = _gn(ag, p + ".gn", x, C)
        h = conv(p + ".proj_in", h, C, 1)
        hs = ag.unary(p + ".to_seq", h, save="none", shape=(Bx, L, C))
        n1 = _ln(ag, p + ".ln1", hs, C)
        hs = ag.add(p + ".sa.res", attn(p + ".sa", n1, n1, C, False), hs)
        n2 = _ln(ag, p + ".ln2", hs, C)
        hs = ag.add(p + ".ca.res", attn(p + ".ca", n2, ctx, C, True), hs)
        n3 = _ln(ag, p + ".ln3", hs, C)
        w1 = ag.param(p + ".ff.w1", (C, 8 * C))
        g = ag.matmul(p + ".ff.fc1", n3, w1, (Bx, L, 8 * C))
        a = ag.unary(p + ".ff.half_a", g, save="none", shape=(Bx, L, 4 * C))
        gt = ag.unary(p + ".ff.half_g", g, save="none", shape=(Bx, L, 4 * C))
        gt = ag.unary(p + ".ff.gelu", gt, save="x", flops_per=8.0)
        ff = ag.binary(p + ".ff.geglu", a, gt)
        w2 = ag.param(p + ".ff.w2", (4 * C, C))
        ff = ag.matmul(p + ".ff.fc2", ff, w2, (Bx, L, C))
        hs = ag.add(p + ".ff.res", ff, hs)
        h = ag.unary(p + ".to_img", hs, save="none", shape=(Bx, C, Hh, Ww))
        h = conv(p + ".proj_out", h, C, 1)
        return ag.add(p + ".res", h, x)

    h = conv("conv_in", x, chans[0], 3)
    skips = [h]
    for lvl, C in enumerate(chans):
        for bi in range(down_blocks):
            h = resblock(f"down{lvl}.res{bi}", h, C)
            if lvl < 3:
                h = transformer_block(f"down{lvl}.attn{bi}", h)
            skips.append(h)
        if lvl < 3:
            h = conv(f"down{lvl}.downsample", h, C, 3, stride=2)
            skips.append(h)
    h = resblock("mid.res0", h, chans[-1])
    h = transformer_block("mid.attn", h)
    h = resblock("mid.res1", h, chans[-1])
    for lvl in reversed(range(len(chans))):
        C = chans[lvl]
        for bi in range(up_blocks):
            s = skips.pop()
            hc = ag.op(f"up{lvl}.cat{bi}", [h, s], (B, h.shape[1] + s.shape[1], h.shape[2], h.shape[3]),
                       numel(h.shape) + numel(s.shape),
                       lambda ag_, dy, out, ins, _n=f"up{lvl}.cat{bi}": [
                           (t, ag_._g(_n + f".d{j}", [dy], t, numel(t.shape))) for j, t in enumerate(ins) if t.grad])
            h = resblock(f"up{lvl}.res{bi}", hc, C)
            if lvl < 3:
                h = transformer_block(f"up{lvl}.attn{bi}", h)
        if lvl > 0:
            up = ag.unary(f"up{lvl}.upsample", h, save="none",
                          shape=(B, C, h.shape[2] * 2, h.shape[3] * 2))
            h = conv(f"up{lvl}.upconv", up, C, 3)
    h = _gn(ag, "out.gn", h, chans[0])
    h = ag.unary("out.silu", h, save="x", flops_per=4.0)
    h = conv("conv_out", h, 4, 3)
    noise = ag.input("noise", h.shape, kind="label")
    loss = ag.loss("mse", h, noise)
    ag.backward(loss)
    return b
