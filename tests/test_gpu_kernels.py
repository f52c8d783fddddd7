"""GPU parity of every hot-path kernel (K1-K9, K11 of SURVEY §2.2) against
the CPU oracle (oracle/model.py) or the plain definition of the op (a
matmul in fp64), on identical seeded inputs, through the C ABI
(include/mobius_kernels.h).  Shapes span several tiles plus ragged tails.

Tolerances (norm-wise ||a-b||/||b||, reading #20): bf16 outputs 1e-2 (one
bf16 rounding of the output ~ 2^-9 plus fp32 accumulation), fp32 outputs
of bf16 products 1e-4, fp32 debug path 1e-5 per kernel; the block and
step-level tests use north_star's 2e-2 (bf16) / 1e-4 (fp32).
"""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import synth  # noqa: E402
from oracle import model as om  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, F32, kt  # noqa: E402

DEV = "cuda:0"


def rel(a, b):
    a = np.asarray(a, dtype=np.float64).reshape(-1)
    b = np.asarray(b, dtype=np.float64).reshape(-1)
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def to_dev(x, dtype):
    t = torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).to(DEV)
    return t.to(torch.bfloat16) if dtype == BF16 else t


def from_dev(t):
    return t.float().cpu().numpy()


def rnd(dtype, x):
    return synth.round_bf16(x) if dtype == BF16 else x.astype(np.float32)


RNG = np.random.default_rng(1)


def randn(*shape, scale=1.0):
    return (RNG.standard_normal(shape) * scale).astype(np.float32)


# ------------------------------------------------------------------ GEMM
# all dims multiples of 8 (TMA: 16-byte row strides), none a multiple of every tile size
# (512, 1600, 320) / (520, 384, 136): 2-CTA tiles whose ragged last column
# (64 / 128 wide) runs as an N = 128 MMA; (640, 392, 256): a 136-wide one (full width)
GEMM_SHAPES = [(256, 256, 256), (200, 320, 192), (136, 64, 64), (384, 96, 1000), (128, 512, 128),
               (344, 264, 136), (1024, 1024, 512), (512, 1600, 320), (520, 384, 136), (640, 392, 256)]


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("a_mn", [False, True])
@pytest.mark.parametrize("b_mn", [False, True])
@pytest.mark.parametrize("shape", GEMM_SHAPES)
def test_gemm_layouts(dtype, a_mn, b_mn, shape):
    M, N, K = shape
    A = rnd(dtype, randn(M, K))
    B = rnd(dtype, randn(N, K))
    ref = A.astype(np.float64) @ B.astype(np.float64).T
    tA = to_dev(A.T.copy() if a_mn else A, dtype)
    tB = to_dev(B.T.copy() if b_mn else B, dtype)
    for c_f32 in ([False, True] if dtype == BF16 else [False]):
        tC = torch.zeros((M, N), device=DEV, dtype=torch.float32 if (c_f32 or dtype == F32) else torch.bfloat16)
        kt.gemm(dtype, M, N, K, tA, M if a_mn else K, a_mn, tB, N if b_mn else K, b_mn, tC, N, c_f32=c_f32)
        torch.cuda.synchronize()
        tol = 1e-2 if (dtype == BF16 and not c_f32) else (1e-4 if dtype == BF16 else 1e-5)
        assert rel(from_dev(tC), ref) < tol, (shape, a_mn, b_mn, c_f32)


# Stream-K tail of the 2-CTA kernel (long K only): shapes whose last wave is
# partial over the 74 SM pairs (8192x1600 = 224 tiles -> 2 full waves + 76
# split tiles; 2000x1000 = 32 tiles, each split over up to 4 pairs, ragged
# M, N and K; 1600x6400 = 175 tiles, the fc1 dW shape).
SK_SHAPES = [(8192, 1600, 6400), (2000, 1000, 4104), (1600, 6400, 8192)]


@pytest.mark.parametrize("shape", SK_SHAPES)
@pytest.mark.parametrize("a_mn,b_mn", [(False, True), (True, True), (False, False)])
def test_gemm_stream_k(shape, a_mn, b_mn):
    M, N, K = shape
    g = torch.Generator(device=DEV).manual_seed(7)
    A = torch.randn(M, K, device=DEV, generator=g).to(torch.bfloat16)
    B = torch.randn(N, K, device=DEV, generator=g).to(torch.bfloat16)
    bias = torch.randn(N, device=DEV, generator=g).to(torch.bfloat16)
    R = torch.randn(M, N, device=DEV, generator=g).to(torch.bfloat16)
    ref = A.double() @ B.double().T
    tA = A.T.contiguous() if a_mn else A
    tB = B.T.contiguous() if b_mn else B

    def run(sk, epi, **kw):
        kt.gemm_config(-1, sk)
        try:
            tC = kw.pop("C")
            kt.gemm(BF16, M, N, K, tA, M if a_mn else K, a_mn, tB, N if b_mn else K, b_mn, tC, N, epi=epi, **kw)
            torch.cuda.synchronize()
        finally:
            kt.gemm_config(-1, -1)
        return tC

    def nrel(a, b):
        return float((a.double() - b).norm() / b.norm())

    # plain store, fp32 out: split-K partial sums reduce to the same product
    c_sk = run(1, 0, C=torch.zeros(M, N, device=DEV), c_f32=True)
    c_dp = run(0, 0, C=torch.zeros(M, N, device=DEV), c_f32=True)
    assert nrel(c_sk, ref) < 1e-5 and nrel(c_dp, ref) < 1e-5
    # deterministic: the reduction order is fixed by segment index
    c_sk2 = run(1, 0, C=torch.zeros(M, N, device=DEV), c_f32=True)
    assert torch.equal(c_sk, c_sk2)
    # fused epilogues run once, on the reduced tile
    out = run(1, 3, C=torch.zeros(M, N, device=DEV, dtype=torch.bfloat16), bias=bias, R=R, ldr=N)
    assert nrel(out, ref + bias.double() + R.double()) < 1e-2
    aux = torch.zeros(M, N, device=DEV, dtype=torch.bfloat16)
    gl = run(1, 2, C=torch.zeros(M, N, device=DEV, dtype=torch.bfloat16), bias=bias, AUX=aux, ldx=N)
    u = ref + bias.double()
    assert nrel(aux, u) < 1e-2
    assert nrel(gl, torch.nn.functional.gelu(u, approximate="tanh")) < 1e-2
    # fp32 accumulate (dW): C = C0 + alpha * acc
    C0 = torch.randn(M, N, device=DEV, generator=g)
    acc = run(1, 5, C=C0.clone(), c_f32=True, accumulate=True, alpha=0.5)
    assert nrel(acc, C0.double() + 0.5 * ref) < 1e-5
    # counters self-reset: a second accumulate launch adds again
    acc2 = run(1, 5, C=acc, c_f32=True, accumulate=True, alpha=0.5)
    assert nrel(acc2, C0.double() + ref) < 1e-5


@pytest.mark.parametrize("dtype", [BF16, F32])
def test_gemm_epilogues(dtype):
    M, N, K = 300, 520, 200
    A = rnd(dtype, randn(M, K))
    B = rnd(dtype, randn(N, K, scale=0.1))
    bias = rnd(dtype, randn(N))
    R = rnd(dtype, randn(M, N))
    acc = A.astype(np.float64) @ B.astype(np.float64).T
    tA, tB = to_dev(A, dtype), to_dev(B.T.copy(), dtype)   # B MN-major as in X W
    tb, tR = to_dev(bias, dtype), to_dev(R, dtype)
    tdt = torch.bfloat16 if dtype == BF16 else torch.float32
    tol = 1e-2 if dtype == BF16 else 1e-5

    def run(epi, **kw):
        tC = torch.zeros((M, N), device=DEV, dtype=kw.pop("cdt", tdt))
        kt.gemm(dtype, M, N, K, tA, K, False, tB, N, True, tC, N, epi=epi, **kw)
        torch.cuda.synchronize()
        return from_dev(tC)

    assert rel(run(1, bias=tb), acc + bias) < tol
    aux = torch.zeros((M, N), device=DEV, dtype=tdt)
    g = run(2, bias=tb, AUX=aux, ldx=N)
    u = acc + bias
    assert rel(from_dev(aux), u) < tol
    assert rel(g, om.gelu_fwd(u)) < tol
    assert rel(run(3, bias=tb, R=tR, ldr=N), acc + bias + R) < tol
    assert rel(run(4, R=tR, ldr=N), acc * om.gelu_grad(R.astype(np.float64))) < tol
    assert abs(rel(run(0, alpha=0.5), 0.5 * acc)) < tol
    # fp32 accumulate: C = C0 + acc
    C0 = randn(M, N)
    tC = torch.from_numpy(C0).to(DEV)
    kt.gemm(dtype, M, N, K, tA, K, False, tB, N, True, tC, N, c_f32=True, epi=5, accumulate=True)
    torch.cuda.synchronize()
    assert rel(from_dev(tC), C0 + acc) < (1e-4 if dtype == BF16 else 1e-5)


@pytest.mark.parametrize("shape", [(300, 520, 200), (200, 192, 64), (2000, 1000, 4104)])
def test_gemm_gelu_bwd_aux(shape):
    """EPI_GELU_BWD with AUX (compact kept activations): C = acc * gelu'(u)
    and AUX = gelu(u), where gelu(u) must be bit-identical to what the
    forward epilogue (EPI_BIAS_GELU) stored for the same bf16 u.  Shapes:
    2-CTA TMA epilogue, 1-CTA epilogue, 2-CTA Stream-K fixup."""
    M, N, K = shape
    g = torch.Generator(device=DEV).manual_seed(11)
    A = (torch.randn(M, K, device=DEV, generator=g) * 0.5).to(torch.bfloat16)
    B = (torch.randn(K, N, device=DEV, generator=g) * 0.1).to(torch.bfloat16)
    bias = (torch.randn(N, device=DEV, generator=g) * 0.5).to(torch.bfloat16)
    # forward: u = A B + bias (AUX), g = gelu(u) (C)
    u = torch.zeros(M, N, device=DEV, dtype=torch.bfloat16)
    g_fwd = torch.zeros(M, N, device=DEV, dtype=torch.bfloat16)
    kt.gemm(BF16, M, N, K, A, K, False, B, N, True, g_fwd, N, epi=2, bias=bias, AUX=u, ldx=N)
    # backward: dU = dY W^T * gelu'(u), g recomputed from u into AUX
    dY = (torch.randn(M, K, device=DEV, generator=g)).to(torch.bfloat16)
    W = (torch.randn(N, K, device=DEV, generator=g) * 0.1).to(torch.bfloat16)
    du = torch.zeros(M, N, device=DEV, dtype=torch.bfloat16)
    g_bwd = torch.zeros(M, N, device=DEV, dtype=torch.bfloat16)
    kt.gemm(BF16, M, N, K, dY, K, False, W, K, False, du, N, epi=4, R=u, ldr=N, AUX=g_bwd, ldx=N)
    torch.cuda.synchronize()
    assert torch.equal(g_bwd, g_fwd)
    ref = (dY.double() @ W.double().T).cpu().numpy() * om.gelu_grad(u.double().cpu().numpy())
    assert rel(from_dev(du), ref) < 1e-2


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("dh", [64, 128])
def test_gemm_attention_views_causal(dtype, dh):
    """Batched head views into a [T, 3h] qkv buffer (4-D tensor maps) and
    the causal tile modes used by K3/K4."""
    mbs, nh, s = 2, 3, 384
    h = nh * dh
    T = mbs * s
    qkv = rnd(dtype, randn(T, 3 * h, scale=0.5))
    tq = to_dev(qkv, dtype)
    q = qkv[:, :h].reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3).astype(np.float64)
    k = qkv[:, h:2 * h].reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3).astype(np.float64)
    v = qkv[:, 2 * h:].reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3).astype(np.float64)
    Sb2, Sb1 = s * s, nh * s * s
    # S = q k^T, skip upper tiles: compare the lower triangle
    tS = torch.full((mbs, nh, s, s), float("nan"), device=DEV, dtype=torch.float32)
    kt.gemm(dtype, s, s, dh, tq, 3 * h, False, tq, 3 * h, False, tS, s, c_f32=True, causal=1, nb1=mbs, nb2=nh,
            abs_=(s * 3 * h, dh), bbs=(s * 3 * h, dh), cbs=(Sb1, Sb2), b_off=h)
    torch.cuda.synchronize()
    S = from_dev(tS)
    ref = q @ k.transpose(0, 1, 3, 2)
    tril = np.tril(np.ones((s, s), dtype=bool))
    assert rel(S[..., tril], ref[..., tril]) < (1e-4 if dtype == BF16 else 1e-5)
    # P lower triangular (zeros above): O = P v with k < m-tile end
    Pm = rnd(dtype, np.where(tril, randn(mbs, nh, s, s, scale=0.05), 0.0))
    tP = to_dev(Pm, dtype)
    tO = torch.zeros((T, h), device=DEV, dtype=torch.bfloat16 if dtype == BF16 else torch.float32)
    kt.gemm(dtype, s, dh, s, tP, s, False, tq, 3 * h, True, tO, h, causal=2, nb1=mbs, nb2=nh, abs_=(Sb1, Sb2),
            bbs=(s * 3 * h, dh), cbs=(s * h, dh), b_off=2 * h)
    torch.cuda.synchronize()
    O = from_dev(tO).reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3)
    tol = 1e-2 if dtype == BF16 else 1e-5
    assert rel(O, Pm.astype(np.float64) @ v) < tol
    # dV = P^T dO with k >= m-tile start (A MN-major)
    dO = rnd(dtype, randn(T, h))
    tdO = to_dev(dO, dtype)
    tdV = torch.zeros((T, h), device=DEV, dtype=tO.dtype)
    kt.gemm(dtype, s, dh, s, tP, s, True, tdO, h, True, tdV, h, causal=3, nb1=mbs, nb2=nh, abs_=(Sb1, Sb2),
            bbs=(s * h, dh), cbs=(s * h, dh))
    torch.cuda.synchronize()
    dO4 = dO.reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3).astype(np.float64)
    dV = from_dev(tdV).reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3)
    assert rel(dV, Pm.astype(np.float64).transpose(0, 1, 3, 2) @ dO4) < tol


# ------------------------------------------------------ row kernels
@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("h", [256, 1600, 5120])
def test_layernorm(dtype, h):
    rows = 37
    x = rnd(dtype, randn(rows, h) * 2 + 0.5)
    g = rnd(dtype, 1 + 0.1 * randn(h))
    b = rnd(dtype, 0.1 * randn(h))
    dy = rnd(dtype, randn(rows, h))
    dres = rnd(dtype, randn(rows, h))
    y_ref, cache = om.layernorm_fwd(x.astype(np.float64), g.astype(np.float64), b.astype(np.float64))
    dx_ref, dg_ref, db_ref = om.layernorm_bwd(dy.astype(np.float64), g.astype(np.float64), cache)
    tx, tg, tb_ = to_dev(x, dtype), to_dev(g, dtype), to_dev(b, dtype)
    ty = torch.empty_like(tx)
    mu = torch.empty(rows, device=DEV)
    rs = torch.empty(rows, device=DEV)
    kt.layernorm_fwd(dtype, tx, tg, tb_, ty, mu, rs, rows, h)
    torch.cuda.synchronize()
    tol = 1e-2 if dtype == BF16 else 1e-5
    assert rel(from_dev(ty), y_ref) < tol
    tdy, tdres = to_dev(dy, dtype), to_dev(dres, dtype)
    tdx = torch.empty_like(tx)
    dg = torch.zeros(h, device=DEV)
    db = torch.zeros(h, device=DEV)
    kt.layernorm_bwd(dtype, tdy, tx, tg, mu, rs, tdres, tdx, dg, db, rows, h)
    torch.cuda.synchronize()
    assert rel(from_dev(tdx), dx_ref + dres) < tol
    assert rel(from_dev(dg), dg_ref) < (1e-4 if dtype == BF16 else 1e-5)
    assert rel(from_dev(db), db_ref) < 1e-5


@pytest.mark.parametrize("env", ["MOBIUS_FLASH_FWD_V1", "MOBIUS_FLASH_BWD_V1"])
def test_attention_v1_fallback(env):
    """The generic (round-2 first session) flash kernels stay selectable at
    dh 64 through MOBIUS_FLASH_FWD_V1 / MOBIUS_FLASH_BWD_V1 = 1 (read once per
    process, so the parity cases run in a child pytest with the variable set)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", os.path.join(root, "tests", "test_gpu_kernels.py"),
                        "-k", "attention_core and 64"], cwd=root, env={**os.environ, env: "1"},
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


@pytest.mark.parametrize("with_res", [True, False])
@pytest.mark.parametrize("rows,h", [(4100, 1600), (301, 8192)])
def test_layernorm_bwd_many_blocks(with_res, rows, h):
    """Fused bf16 LN backward with several row blocks per CTA, a ragged last
    block, with and without the residual gradient, parameter gradients
    accumulated onto non-zero buffers (+=), against the oracle in fp64
    (h 8192: one row per block, four column vectors per thread)."""
    x = rnd(BF16, randn(rows, h) * 2 + 0.5)
    g = rnd(BF16, 1 + 0.1 * randn(h))
    b = rnd(BF16, 0.1 * randn(h))
    dy = rnd(BF16, randn(rows, h))
    dres = rnd(BF16, randn(rows, h))
    _, cache = om.layernorm_fwd(x.astype(np.float64), g.astype(np.float64), b.astype(np.float64))
    dx_ref, dg_ref, db_ref = om.layernorm_bwd(dy.astype(np.float64), g.astype(np.float64), cache)
    tx, tg, tb_ = to_dev(x, BF16), to_dev(g, BF16), to_dev(b, BF16)
    ty = torch.empty_like(tx)
    mu = torch.empty(rows, device=DEV)
    rs = torch.empty(rows, device=DEV)
    kt.layernorm_fwd(BF16, tx, tg, tb_, ty, mu, rs, rows, h)
    tdy, tdres = to_dev(dy, BF16), to_dev(dres, BF16)
    tdx = torch.full_like(tx, float("nan"))
    dg0, db0 = randn(h), randn(h)
    dg = torch.from_numpy(dg0.astype(np.float32)).to(DEV)
    db = torch.from_numpy(db0.astype(np.float32)).to(DEV)
    kt.layernorm_bwd(BF16, tdy, tx, tg, mu, rs, tdres if with_res else None, tdx, dg, db, rows, h)
    torch.cuda.synchronize()
    got = from_dev(tdx)
    want = dx_ref + dres if with_res else dx_ref
    assert np.isfinite(got).all()
    assert rel(got, want) < 1e-2
    assert np.max(np.abs(got - want)) <= 0.05 * np.max(np.abs(want))
    assert rel(from_dev(dg) - dg0, dg_ref) < 1e-4
    assert rel(from_dev(db) - db0, db_ref) < 1e-5


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("s", [128, 384])
def test_softmax_causal(dtype, s):
    B = 3
    S = randn(B, s, s, scale=3.0)
    scale = 1 / math.sqrt(64)
    mask = np.triu(np.ones((s, s), dtype=bool), 1)
    P_ref = om.softmax_rows(np.where(mask, -np.inf, S.astype(np.float64) * scale))
    tS = torch.from_numpy(S).to(DEV)
    tP = torch.full((B, s, s), 7.0, device=DEV, dtype=torch.bfloat16 if dtype == BF16 else torch.float32)
    kt.softmax_fwd(dtype, tS, tP, B, s, scale)
    torch.cuda.synchronize()
    P = from_dev(tP)
    tol = 1e-2 if dtype == BF16 else 1e-5
    tril = ~mask
    assert rel(P[:, tril], P_ref[:, tril]) < tol
    # zeros above the diagonal inside the row's 128-wide tile
    for i in range(s):
        end = min(s, (i // 128 + 1) * 128)
        assert np.all(P[:, i, i + 1:end] == 0)
    # backward
    dP = randn(B, s, s)
    Pq = P.astype(np.float64)
    dS_ref = scale * Pq * (dP - (dP * Pq * tril).sum(-1, keepdims=True)) * tril
    tdP = torch.from_numpy(dP).to(DEV)
    tdS = torch.full_like(tP, 7.0)
    kt.softmax_bwd(dtype, tP, tdP, tdS, B, s, scale)
    torch.cuda.synchronize()
    dS = from_dev(tdS)
    assert rel(dS[:, tril], dS_ref[:, tril]) < tol


@pytest.mark.parametrize("dtype", [BF16, F32])
def test_cross_entropy(dtype):
    mbs, s, V = 2, 64, 512
    rows = mbs * s
    z = rnd(dtype, randn(rows, V, scale=2.0))
    tok = RNG.integers(0, V, size=(mbs, s + 1)).astype(np.int32)
    tgt = tok[:, 1:].reshape(-1)
    ntok = 1000
    zz = z.astype(np.float64)
    m = zz.max(-1, keepdims=True)
    e = np.exp(zz - m)
    lse = (m + np.log(e.sum(-1, keepdims=True)))[:, 0]
    loss_ref = lse - zz[np.arange(rows), tgt]
    dz_ref = e / e.sum(-1, keepdims=True)
    dz_ref[np.arange(rows), tgt] -= 1
    dz_ref /= ntok
    tz = to_dev(z, dtype)
    ttok = torch.from_numpy(tok).to(DEV)
    lr = torch.empty(rows, device=DEV)
    kt.cross_entropy(dtype, tz, ttok, lr, rows, V, s, 1.0 / ntok)
    torch.cuda.synchronize()
    assert rel(from_dev(lr), loss_ref) < (1e-4 if dtype == BF16 else 1e-5)
    assert rel(from_dev(tz), dz_ref) < (1e-2 if dtype == BF16 else 1e-5)


@pytest.mark.parametrize("dtype", [BF16, F32])
def test_embedding(dtype):
    cfg = synth.GPTConfig(n_layers=1, hidden=256, n_heads=4, seq_len=128, vocab=512, micro_batch=3)
    p = {"wte": rnd(dtype, randn(512, 256)), "wpe": rnd(dtype, randn(128, 256))}
    tok = RNG.integers(0, 512, size=(3, 129)).astype(np.int32)
    tok[0, :10] = 7  # repeated tokens exercise the scatter-add
    x_ref, _ = om.embed_fwd(cfg, p, tok[:, :-1])
    ttok = torch.from_numpy(tok).to(DEV)
    twte, twpe = to_dev(p["wte"], dtype), to_dev(p["wpe"], dtype)
    tx = torch.empty((3 * 128, 256), device=DEV, dtype=twte.dtype)
    kt.embed_fwd(dtype, ttok, twte, twpe, tx, 3, 128, 256)
    torch.cuda.synchronize()
    assert rel(from_dev(tx), x_ref) < (1e-2 if dtype == BF16 else 1e-6)
    dx = rnd(dtype, randn(3 * 128, 256))
    g_ref = om.embed_bwd(cfg, {k: v.astype(np.float64) for k, v in p.items()}, dx.astype(np.float64), tok[:, :-1])
    dwte = torch.zeros((512, 256), device=DEV)
    dwpe = torch.zeros((128, 256), device=DEV)
    kt.embed_bwd(dtype, ttok, to_dev(dx, dtype), dwte, dwpe, 3, 128, 256)
    torch.cuda.synchronize()
    assert rel(from_dev(dwte), g_ref["wte"]) < 1e-5
    assert rel(from_dev(dwpe), g_ref["wpe"]) < 1e-5


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("dist", ["uniform", "zipf", "single"])
def test_embedding_bwd_deterministic_large_vocab(dtype, dist):
    """dWte scatter at V = 50304 with uniform, Zipf-skewed (a few ids own
    thousands of positions) and single-id token streams: equal to the fp64
    segment sums; on the fp32 path (ownership split over ~600 CTAs, ragged
    last owner, several scan rounds) bitwise identical across runs (no
    atomics: P:L596-602 synchronous-update reproducibility is checked bit
    for bit there); the bf16 path uses vector reductions."""
    V, h, mbs, s = 50304, 256, 8, 1024
    rng = np.random.default_rng(17)
    if dist == "uniform":
        tok = rng.integers(0, V, size=(mbs, s + 1))
    elif dist == "zipf":
        tok = np.minimum(rng.zipf(1.2, size=(mbs, s + 1)) - 1, V - 1)
    else:
        tok = np.full((mbs, s + 1), V - 1)
    tok = tok.astype(np.int32)
    dx = rnd(dtype, randn(mbs * s, h))
    ids = tok[:, :-1].reshape(-1)
    ref = np.zeros((V, h))
    np.add.at(ref, ids, dx.astype(np.float64))
    ttok = torch.from_numpy(tok).to(DEV)
    tdx = to_dev(dx, dtype)
    outs = []
    for _ in range(2):
        dwte = torch.zeros((V, h), device=DEV)
        dwpe = torch.zeros((s, h), device=DEV)
        kt.embed_bwd(dtype, ttok, tdx, dwte, dwpe, mbs, s, h, V)
        torch.cuda.synchronize()
        outs.append(dwte.cpu().numpy())
    if dtype == F32:
        assert np.array_equal(outs[0], outs[1])
    touched = np.unique(ids)
    # fp32 sums of up to mbs*s = 8192 rows in position order: |err| <~ sqrt(n) u |sum|
    assert rel(outs[0][touched], ref[touched]) < 1e-5
    untouched = np.setdiff1d(np.arange(V), touched)
    assert not outs[0][untouched].any()


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("rows,n", [(32768, 1600), (4096, 6400), (1000, 520), (333, 64)])
def test_colsum_deterministic(dtype, rows, n):
    """Column sums (bias / LayerNorm-parameter gradients) at the bench's
    shapes: fp64 reference within fp32 rounding and bitwise identical over
    repeated launches (fixed CTA-order reduction, no atomics)."""
    X = rnd(dtype, randn(rows, n))
    tX = to_dev(X, dtype)
    outs = []
    for _ in range(3):
        t = torch.zeros(n, device=DEV)
        kt.colsum(dtype, tX, n, rows, n, t)
        torch.cuda.synchronize()
        outs.append(t.cpu().numpy())
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])
    assert rel(outs[0], X.astype(np.float64).sum(0)) < 1e-5


@pytest.mark.parametrize("dtype", [BF16, F32])
def test_colsum(dtype):
    X = rnd(dtype, randn(1000, 520))
    out0 = randn(520)
    t = torch.from_numpy(out0.copy()).to(DEV)
    kt.colsum(dtype, to_dev(X, dtype), 520, 1000, 520, t)
    torch.cuda.synchronize()
    assert rel(from_dev(t), out0 + X.astype(np.float64).sum(0)) < 1e-5


# --------------------------------------------------------- block level
@pytest.mark.parametrize("dtype,tol,wscale", [(BF16, 2e-2, 1.0), (BF16, 5e-2, 3.0), (F32, 1e-4, 3.0)])
@pytest.mark.parametrize("h,nh,s,mbs", [(256, 4, 128, 2), (256, 2, 256, 1), (384, 3, 384, 1)])
def test_block_fwd_bwd(dtype, tol, wscale, h, nh, s, mbs):
    """One block fwd+bwd vs the fp64 oracle.  wscale=1 is the O-1 init
    (with perturbed LN/bias terms); wscale=3 sharpens the attention as a
    stress case (bf16 tolerance widened to 5e-2 for it: bf16 P/dS)."""
    cfg = synth.GPTConfig(n_layers=4, hidden=h, n_heads=nh, seq_len=s, vocab=64, micro_batch=mbs)
    flat = synth.perturb_norm_params(cfg, synth.gen_params(cfg), scale=0.2)
    offs = cfg.layer_offsets()
    wb = rnd(dtype, flat[offs[1]:offs[2]] * wscale)
    p = om.unpack_layer(cfg, np.concatenate([flat[:offs[1]], wb.astype(np.float32), flat[offs[2]:]]), 1)
    p64 = {k: v.astype(np.float64) for k, v in p.items()}
    T = mbs * s
    x = rnd(dtype, randn(T, h))
    dy = rnd(dtype, randn(T, h))
    y_ref, cache = om.block_fwd(cfg, p64, x.astype(np.float64), mbs)
    dx_ref, g_ref = om.block_bwd(cfg, p64, dy.astype(np.float64), cache, mbs)
    tw = to_dev(wb, dtype)
    tx, tdy = to_dev(x, dtype), to_dev(dy, dtype)
    ty = torch.empty_like(tx)
    tdx = torch.empty_like(tx)
    grads = torch.zeros(wb.size, device=DEV)
    kt.block(dtype, h, nh, s, mbs, tw, tx, ty, tdy, tdx, grads)
    torch.cuda.synchronize()
    G = from_dev(grads)
    pos = 0
    errs = {"y": rel(from_dev(ty), y_ref), "dx": rel(from_dev(tdx), dx_ref)}
    for name, shape, _ in cfg.layer_specs(1):
        n = int(np.prod(shape))
        errs[name] = rel(G[pos:pos + n], g_ref[name])
        pos += n
    print(errs)
    assert max(errs.values()) < tol, errs


@pytest.mark.parametrize("dtype", [BF16, F32])
@pytest.mark.parametrize("mbs,s,nh,dh", [(2, 128, 2, 64), (1, 384, 3, 64), (2, 256, 2, 128), (1, 1024, 2, 64),
                                         (4, 1024, 25, 64), (2, 1024, 12, 128), (1, 2048, 3, 64)])
def test_attention_core(dtype, mbs, s, nh, dh):
    """Causal attention fwd+bwd (fused tcgen05 flash kernels on the bf16 path)
    vs the oracle's attention_fwd / attention_bwd in fp64."""
    h = nh * dh
    T = mbs * s
    qkv = rnd(dtype, randn(T, 3 * h, scale=1.0))
    dout = rnd(dtype, randn(T, h))
    o_ref, cache = om.attention_fwd(qkv.astype(np.float64), mbs, s, nh)
    dqkv_ref = om.attention_bwd(dout.astype(np.float64), cache, mbs, s, nh)
    tq = to_dev(qkv, dtype)
    to = torch.zeros((T, h), device=DEV, dtype=tq.dtype)
    tdo = to_dev(dout, dtype)
    tdq = torch.full((T, 3 * h), float("nan"), device=DEV, dtype=tq.dtype)
    kt.attention(dtype, mbs, s, nh, dh, tq, to, tdo, tdq)
    torch.cuda.synchronize()
    tol = 2e-2 if dtype == BF16 else 1e-5
    d = from_dev(tdq)
    errs = {"o": rel(from_dev(to), o_ref)}
    for part, name in ((0, "dq"), (1, "dk"), (2, "dv")):
        errs[name] = rel(d[:, part * h:(part + 1) * h], dqkv_ref[:, part * h:(part + 1) * h])
    assert max(errs.values()) < tol, errs
