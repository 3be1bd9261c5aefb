"""The data-parallel gradient all-reduce executed on
one B200: a context with ``comm_force = 1`` builds a real NCCL communicator
(1 rank: this pod leases one GPU, and NCCL refuses two ranks on one device)
and runs exactly the multi-GPU code path -- the per-layer-bucket
ncclAllReduce on the high-priority comm stream gated by the wgrad events, the
fused per-bucket AdamW behind each all-reduce with the 1/world scale, the
scalar-loss all-reduce, and the cross-rank plan-hash check.

With one rank the sum is the identity, so everything must be BITWISE equal to
the communicator-free path, whose results the oracle parity tests pin.  The
N-rank semantics (mean of per-rank gradients == gradient of the concatenated
batch, c-J) are pinned on the oracle with a real 2-rank gloo group
(tests/test_oracle_dp.py)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import memsim as om
from oracle import model as omodel
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

CASES = {
    "mc-bf16": wl.small_config("bert-base", n_layers=3, hidden=128, heads=2, ffn=256, vocab=500,
                               max_pos=64, n_seqs=8, seq_lo=8, seq_hi=40, pad=8),
    "lm-gpt2-bf16": wl.small_config("gpt2-medium", n_layers=2, hidden=128, heads=2, ffn=256, vocab=600,
                                    max_pos=128, n_seqs=3, seq_lo=40, seq_hi=120, pad=8, pad_id=599,
                                    cls_id=599, sep_id=599),
    "bert-base-full": wl.small_config("bert-base", n_layers=4),
}


def ctx_for(cfg, **kw):
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    budget = om.no_ckpt_peak(om.sizes(cfg, cfg.n_seqs, cfg.max_seq))
    slab = torch.empty(budget, dtype=torch.uint8, device="cuda")
    return mb.Mimose(cfg, budget, slab=slab, stream=torch.cuda.current_stream(), **kw), slab


def steps(cfg, params, fused, n=3, **kw):
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    ctx, slab = ctx_for(cfg, **kw)
    ctx.set_params(wl.pack_params(cfg, params))
    if fused:
        ctx.set_optimizer(lr=1e-3, wd=0.01, fused=True)
    losses, grads = [], []
    for i, L in enumerate([cfg.seq_hi, cfg.seq_lo + 3, (cfg.seq_lo + cfg.seq_hi) // 2][:n]):
        b = wl.make_batch(cfg, L, seed=60 + i)
        p = mb.Plan()
        p.drop_mask = 1                                   # layer 0 recomputed
        losses.append(ctx.forward(ctx.host_batch(b), p))
        ctx.backward()
        torch.cuda.synchronize()
        grads.append(ctx.get_grads())
        ctx.step(lr=1e-3, wd=0.01)
    torch.cuda.synchronize()
    out = dict(losses=losses, grads=grads, params=ctx.get_params(), stats=ctx.stats())
    ctx.close()
    return out


@pytest.mark.parametrize("case", list(CASES))
@pytest.mark.parametrize("fused", [False, True])
@pytest.mark.parametrize("zero1", [0, 1])
def test_nccl_allreduce_path_bitwise(case, fused, zero1):
    """zero1 = 1: the ZeRO-1 path -- per-bucket ncclReduceScatter,
    AdamW on this rank's shard of master / m / v, ncclAllGather of the bf16
    weights -- which at one rank must equal the unsharded step bit for bit."""
    cfg = CASES[case]
    params = wl.init_params(cfg, parity=True, seed=4)
    ref = steps(cfg, params, fused)
    got = steps(cfg, params, fused, comm_force=1, check_plans=1, zero1=zero1)
    st = got["stats"]
    assert st["comm_nranks"] == 1 and ref["stats"]["comm_nranks"] == 0
    # one bucket per encoder layer + head + embedding, every backward
    assert st["allreduce_calls"] == 3 * (cfg.n_layers + 2) and ref["stats"]["allreduce_calls"] == 0
    n_params_padded = sum(-(-int(np.prod(s)) // 64) * 64 for _, s in wl.param_spec(cfg))
    assert st["allreduce_bytes"] == 3 * 4 * n_params_padded
    assert st["plan_checks"] == 3
    assert got["losses"] == ref["losses"]                  # loss all-reduce (avg over 1 rank)
    for g0, g1 in zip(ref["grads"], got["grads"]):
        assert np.array_equal(g0, g1)
    assert np.array_equal(ref["params"], got["params"])    # AdamW after the all-reduce, 1/world


def test_nccl_path_against_oracle():
    """The all-reduced gradients of a step are the oracle's (plain fp64 step on
    the bf16-rounded weights, same Philox masks) within the c-K bound."""
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    cfg = CASES["mc-bf16"]
    params = wl.init_params(cfg, parity=True, seed=4)
    ctx, slab = ctx_for(cfg, comm_force=1)
    ctx.set_params(wl.pack_params(cfg, params))
    b = wl.make_batch(cfg, cfg.seq_hi, seed=61)
    p = mb.Plan()
    p.drop_mask = 0b101
    loss = ctx.forward(ctx.host_batch(b), p)
    ctx.backward()
    torch.cuda.synchronize()
    g = wl.unpack_params(cfg, ctx.get_grads())
    assert ctx.stats()["allreduce_calls"] == cfg.n_layers + 2
    ctx.close()
    W = {k: torch.tensor(v).bfloat16().double().numpy() for k, v in params.items()}
    ref_loss, G = omodel.train_step_grads(cfg, W, b, wl.dropout_seed(cfg), 1)
    assert abs(loss - ref_loss) <= 2e-2 * max(1.0, abs(ref_loss))
    for k in G:
        if k == "cls.b":          # provably zero (MC CE is shift invariant over choices)
            continue
        err = np.abs(g[k] - G[k]).max() / np.abs(G[k]).max()
        assert err <= 2e-2, (k, err)


def test_plan_check_detects_mismatch_is_noop_single_rank():
    """With one rank every hash matches its own: the check passes and counts."""
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    cfg = CASES["mc-bf16"]
    ctx, slab = ctx_for(cfg, comm_force=1, check_plans=1, nccl_max_ctas=-1)
    ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
    b = wl.make_batch(cfg, 20, seed=3)
    ctx.forward(ctx.host_batch(b), None, False)
    ctx.backward()
    ctx.step()
    assert ctx.stats()["plan_checks"] == 1
    ctx.close()


def test_zero1_needs_a_communicator():
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    with pytest.raises(mb.MimoseError):
        ctx_for(CASES["mc-bf16"], zero1=1)
