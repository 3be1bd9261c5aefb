"""The library's bf16 GEMMs (tcgen05/TMEM/TMA and SIMT) against a plain PyTorch
fp32 reference of the same op: every operand-major combination the step uses
(forward NT, dgrad NN, wgrad TN), ragged M/N/K tails, bias epilogue, split-K."""
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def mb():
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding
    return binding


SHAPES = [(256, 256, 128), (300, 200, 136), (2048, 768, 768), (1000, 2304, 768), (768, 3072, 520), (128, 128, 64)]


def operands(M, N, K, a_mn, b_mn, seed=0):
    g = torch.Generator(device="cuda").manual_seed(seed)
    A = torch.randn(M, K, device="cuda", generator=g).bfloat16()
    B = torch.randn(N, K, device="cuda", generator=g).bfloat16()
    # storage: K-major = [rows, K] row-major; MN-major = [K, rows] row-major
    As = A.t().contiguous() if a_mn else A.contiguous()
    Bs = B.t().contiguous() if b_mn else B.contiguous()
    a_sm, a_sk = (1, M) if a_mn else (K, 1)
    b_sn, b_sk = (1, N) if b_mn else (K, 1)
    return A, B, As, Bs, a_sm, a_sk, b_sn, b_sk


SHAPES += [(2048, 3072, 768), (512, 768, 3072), (4096, 2304, 768)]   # BN=256 persistent tiles


@pytest.fixture(params=[1, 14, 13, 2, 0], ids=["persistent", "stream-k", "persistent-bn64", "cta-pair", "tile-per-cta"])
def gemm_mode(request):
    mb().debug_options(gemm_mode=request.param)
    yield request.param
    mb().debug_options(gemm_mode=1)


@pytest.mark.parametrize("use_tc", [True, False])
@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 1)])
@pytest.mark.parametrize("shape", SHAPES)
def test_gemm_f32_out(shape, a_mn, b_mn, use_tc, gemm_mode):
    if not use_tc and gemm_mode != 1:
        pytest.skip("SIMT path does not depend on the tcgen05 mode")
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, a_mn, b_mn)
    C = torch.full((M, N), float("nan"), device="cuda")
    mb().debug_gemm(6, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, use_tc=use_tc)
    torch.cuda.synchronize()
    ref = A.float() @ B.float().t()
    err = (C - ref).abs().max().item() / ref.abs().max().item()
    assert err < 1e-5, err


@pytest.mark.parametrize("shape", [(300, 200, 136), (2048, 768, 768), (2048, 3072, 768)])
def test_gemm_bias_bf16_out(shape, gemm_mode):
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 0, 0, seed=1)
    bias = torch.randn(N, device="cuda").bfloat16()
    C = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
    mb().debug_gemm(1, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, bias=bias)
    torch.cuda.synchronize()
    ref = A.float() @ B.float().t() + bias.float()
    err = (C.float() - ref).abs().max().item() / ref.abs().max().item()
    assert err < 1e-2, err


@pytest.mark.parametrize("split", [2, 3, 4])
def test_gemm_split_k(split, gemm_mode):
    M, N, K = 768, 768, 1000            # wgrad-like: TN, K = tokens
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 1, 1, seed=2)
    C = torch.zeros(split, M, N, device="cuda")
    mb().debug_gemm(6, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, split=split)
    torch.cuda.synchronize()
    ref = A.float() @ B.float().t()
    err = (C.sum(0) - ref).abs().max().item() / ref.abs().max().item()
    assert err < 1e-5, err


@pytest.mark.parametrize("shape,split", [((768, 3072, 5120), 2), ((3072, 768, 4096), 2), ((2304, 768, 2048), 3),
                                         ((768, 768, 5120), 5), ((1024, 1024, 1536), 4), ((640, 512, 777), 2)])
def test_gemm_fused_splitk(shape, split):
    """wgrad-shaped TN GEMM with the in-kernel fused split-K: matches the fp32
    reference, and two launches are bitwise identical (fixed reduction order)."""
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 1, 1, seed=3)
    ws = torch.full(((split - 1) * M * N,), float("nan"), device="cuda")
    outs = []
    for _ in range(2):
        C = torch.full((M, N), float("nan"), device="cuda")
        mb().debug_gemm_ex(6, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, C2=ws, split=-split)
        torch.cuda.synchronize()
        outs.append(C)
    ref = A.float() @ B.float().t()
    err = (outs[0] - ref).abs().max().item() / ref.abs().max().item()
    assert err < 1e-5, err
    assert torch.equal(outs[0], outs[1])


@pytest.mark.parametrize("shape", [(640, 3072, 768), (2048, 3072, 768)])
def test_gemm_gelu_epilogues(shape, gemm_mode):
    """EPI_BIAS_GELU (u = acc + b, g = gelu(u)) and EPI_GELU_BWD (acc * gelu'(u))
    against the exact erf-GELU in fp32 (torch): u to bf16 rounding, g and the
    gradient within one bf16 ulp of the exact value (the tcgen05 epilogue uses
    the single-MUFU tanh form, |error| < 1e-3, DESIGN reading R-G)."""
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 0, 0, seed=4)
    bias = torch.randn(N, device="cuda").bfloat16()
    U = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
    Gk = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
    A = A / 8
    As = As / 8
    mb().debug_gemm_ex(2, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, U, N, C2=Gk, bias=bias)
    torch.cuda.synchronize()
    ref_u = A.float() @ B.float().t() + bias.float()
    assert ((U.float() - ref_u).abs().max() / ref_u.abs().max()).item() < 1e-2
    g_exact = torch.nn.functional.gelu(U.float())
    assert ((Gk.float() - g_exact).abs() <= 2.0 ** -7 * g_exact.abs().clamp_min(1.0)).all()
    # backward epilogue: D = acc * gelu'(aux), aux = U
    D = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
    mb().debug_gemm_ex(4, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, D, N, aux=U, ldx=N)
    torch.cuda.synchronize()
    u = U.float().requires_grad_(True)
    torch.nn.functional.gelu(u).backward(torch.ones_like(u))
    ref_d = (A.float() @ B.float().t()) * u.grad
    err = ((D.float() - ref_d).abs().max() / ref_d.abs().max()).item()
    assert err < 1e-2, err


SK_SHAPES = [(300, 256, 1000), (2048, 768, 3072), (768, 3072, 5120), (1000, 2304, 136), (5120, 768, 768),
             (130, 384, 4160)]


@pytest.mark.parametrize("epi", [1, 2, 3, 4, 5, 6])
@pytest.mark.parametrize("shape", SK_SHAPES)
def test_gemm_stream_k(shape, epi):
    """Deterministic stream-K (gemm_mode 14 forces it): every epilogue matches
    the data-parallel persistent kernel (mode 12: same 128 x 256 tiles, one CTA
    per tile) up to fp32 summation order, and two launches are bitwise equal
    (the (tile, k-block) ranges and the partial order are fixed by the shape)."""
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, int(epi == 6), int(epi in (4, 5, 6)), seed=5)
    As = As / 8
    g = torch.Generator(device="cuda").manual_seed(6)
    bias = torch.randn(N, device="cuda", generator=g).bfloat16()
    res_b = torch.randn(M, N, device="cuda", generator=g).bfloat16()
    res_f = torch.randn(M, N, device="cuda", generator=g)
    f32_out = epi in (3, 5, 6)

    def run(mode):
        mb().debug_options(gemm_mode=mode)
        C = torch.full((M, N), float("nan"), device="cuda", dtype=torch.float32 if f32_out else torch.bfloat16)
        C2 = torch.full((M, N), float("nan"), device="cuda", dtype=torch.bfloat16)
        kw = {}
        if epi in (1, 2, 3):
            kw["bias"] = bias
        if epi == 2:
            kw["C2"] = C2
        if epi == 3:
            kw.update(res=res_b, ldr=N)
        if epi == 4:
            kw.update(aux=res_b, ldx=N)
        if epi == 5:
            C.copy_(res_f)
            kw.update(res=C, ldr=N)    # res aliases C, as in the step
        mb().debug_gemm_ex(epi, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, **kw)
        torch.cuda.synchronize()
        return C.float(), C2.float()

    try:
        ref, ref2 = run(12)
        a1, a2 = run(14)
        b1, b2 = run(14)
    finally:
        mb().debug_options(gemm_mode=1)
    tol = 1e-5 if f32_out else 2e-2
    err = ((a1 - ref).abs().max() / ref.abs().max()).item()
    assert err < tol, err
    assert torch.equal(a1, b1)
    if epi == 2:
        assert ((a2 - ref2).abs().max() / ref2.abs().max()).item() < 2e-2
        assert torch.equal(a2, b2)


@pytest.mark.parametrize("pair", [((768, 3072, 5120), (3072, 768, 5120)), ((768, 3072, 1000), (3072, 768, 1000)),
                                  ((296, 512, 136), (1000, 256, 136))])
def test_gemm_grouped_wgrad(pair):
    """Two wgrad-shaped (TN) fp32 GEMMs in one grouped launch are bitwise equal
    to the same problems launched alone with the same 128 x 256 tiles."""
    outs, refs = [], []
    ops = []
    for i, (M, N, K) in enumerate(pair):
        A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 1, 1, seed=20 + i)
        ops.append((M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk))
        refs.append(A.float() @ B.float().t())
    C = [torch.full((o[0], o[1]), float("nan"), device="cuda") for o in ops]
    mb().debug_gemm_grouped(ops[0], C[0], ops[1], C[1])
    torch.cuda.synchronize()
    mb().debug_options(gemm_mode=12)          # separate persistent launches, 256-wide tiles
    try:
        for o, ref, c in zip(ops, refs, C):
            M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk = o
            alone = torch.full((M, N), float("nan"), device="cuda")
            mb().debug_gemm(6, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, alone, N)
            torch.cuda.synchronize()
            assert torch.equal(c, alone)
            assert ((c - ref).abs().max() / ref.abs().max()).item() < 1e-5
    finally:
        mb().debug_options(gemm_mode=1)
