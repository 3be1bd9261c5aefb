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


@pytest.fixture(params=[1, 12, 15, 17], ids=["persistent", "persistent-bn256", "persistent-lsu-store", "cta-pair"])
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


@pytest.mark.parametrize("mode", [1, 15])
@pytest.mark.parametrize("pair", [((768, 3072, 5120), (3072, 768, 5120)), ((768, 3072, 1000), (3072, 768, 1000)),
                                  ((296, 512, 136), (1000, 256, 136))])
def test_gemm_grouped_wgrad(pair, mode):
    """Two wgrad-shaped (TN) fp32 GEMMs in one grouped launch are bitwise equal
    to the same problems launched alone with the same 128 x 256 tiles."""
    outs, refs = [], []
    ops = []
    for i, (M, N, K) in enumerate(pair):
        A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 1, 1, seed=20 + i)
        ops.append((M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk))
        refs.append(A.float() @ B.float().t())
    C = [torch.full((o[0], o[1]), float("nan"), device="cuda") for o in ops]
    mb().debug_options(gemm_mode=mode)
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


@pytest.mark.parametrize("epi", [0, 1, 2, 3, 4, 5, 6, 8, 9, 10])
@pytest.mark.parametrize("shape", [(300, 776, 136), (2100, 3072, 768), (1000, 768, 3072)])
def test_tma_store_epilogues_bitwise(epi, shape):
    """The TMA-store epilogue (default: fragments written through swizzled smem
    by cp.async.bulk.tensor, rows >= M clipped by the unit) stores exactly what
    the LSU-store epilogue (gemm mode 15) stores, for every epilogue, with ragged M and
    an N tail (776 = 24 full 32-column chunks + 8 columns on the scalar path)."""
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, 0, 0, seed=30 + epi)
    bf, f32 = torch.bfloat16, torch.float32
    out_f32 = epi in (3, 5, 6, 10)
    g = torch.Generator(device="cuda").manual_seed(7)
    bias = torch.randn(N, device="cuda", generator=g).to(bf)
    res = torch.randn(M, N, device="cuda", generator=g)
    aux = torch.randn(M, N, device="cuda", generator=g).to(bf)
    outs = []
    for mode in (15, 1):
        C = torch.full((M, N), float("nan"), device="cuda", dtype=f32 if out_f32 else bf)
        C2 = torch.full((M, N), float("nan"), device="cuda", dtype=bf)
        kw = dict(bias=bias)
        if epi in (2, 8):
            kw["C2"] = C2
        if epi == 3:
            kw.update(res=res.to(bf), ldr=N)
        if epi in (5, 10):
            kw.update(res=res, ldr=N)
        if epi in (4, 9):
            kw.update(aux=aux, ldx=N)
        mb().debug_options(gemm_mode=mode)
        try:
            mb().debug_gemm_ex(epi, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, **kw)
            torch.cuda.synchronize()
        finally:
            mb().debug_options(gemm_mode=1)
        outs.append((C, C2))
    assert not torch.isnan(outs[0][0].float()).any()
    assert torch.equal(outs[0][0], outs[1][0])
    if epi in (2, 8):
        assert torch.equal(outs[0][1], outs[1][1])


@pytest.mark.parametrize("epi", [0, 2, 3, 4, 5, 6])
@pytest.mark.parametrize("shape,majors", [((300, 768, 136), (0, 0)), ((2100, 3072, 768), (0, 0)),
                                          ((1000, 768, 3072), (0, 1)), ((768, 3072, 1000), (1, 1))])
def test_cta_pair_bitwise(epi, shape, majors):
    """The CTA-pair kernel (gemm mode 17: cta_group::2, 256 x 256 tiles over two
    SMs) accumulates every output element over K in the same order as the
    single-CTA kernel with 256-wide tiles (mode 12), so every epilogue's output
    is bitwise equal -- with M not a multiple of 256 (the second CTA's rows
    partly or wholly past M) and both operand majors."""
    if majors != (0, 0) and epi not in (6,):
        pytest.skip("MN-major operands: the weight-gradient (fp32) epilogue")
    M, N, K = shape
    A, B, As, Bs, a_sm, a_sk, b_sn, b_sk = operands(M, N, K, *majors, seed=40 + epi)
    bf, f32 = torch.bfloat16, torch.float32
    out_f32 = epi in (3, 5, 6)
    g = torch.Generator(device="cuda").manual_seed(9)
    bias = torch.randn(N, device="cuda", generator=g).to(bf)
    res = torch.randn(M, N, device="cuda", generator=g)
    aux = torch.randn(M, N, device="cuda", generator=g).to(bf)
    outs = []
    for mode in (12, 17):
        C = torch.full((M, N), float("nan"), device="cuda", dtype=f32 if out_f32 else bf)
        C2 = torch.full((M, N), float("nan"), device="cuda", dtype=bf)
        kw = dict(bias=bias)
        if epi == 2:
            kw["C2"] = C2
        if epi == 3:
            kw.update(res=res.to(bf), ldr=N)
        if epi == 5:
            kw.update(res=res, ldr=N)
        if epi == 4:
            kw.update(aux=aux, ldx=N)
        mb().debug_options(gemm_mode=mode)
        try:
            mb().debug_gemm_ex(epi, M, N, K, As, a_sm, a_sk, Bs, b_sn, b_sk, C, N, **kw)
            torch.cuda.synchronize()
        finally:
            mb().debug_options(gemm_mode=1)
        outs.append((C, C2))
    assert not torch.isnan(outs[0][0].float()).any()
    assert torch.equal(outs[0][0], outs[1][0])
    if epi == 2:
        assert torch.equal(outs[0][1], outs[1][1])
