"""The phase-word hooks on a real PyTorch training loop, and
the paper's semantics check (exact floating-point loss match
with vs without JIT recovery, under determinism): two data-parallel replicas
train in lockstep; one fails inside its optimizer step (DIRTY); the other is
selected, captured and restored into a fresh replacement, which then trains
on with exactly the same losses as the surviving replica."""
import os
import shutil
import uuid

import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    return jitc


def _model(seed):
    torch.manual_seed(seed)
    return torch.nn.Sequential(torch.nn.Linear(256, 512), torch.nn.GELU(), torch.nn.Linear(512, 256)).cuda()


def _step(model, opt, x, y):
    opt.zero_grad(set_to_none=False)
    loss = torch.nn.functional.mse_loss(model(x), y)
    loss.backward()
    opt.step()
    return loss.detach()


def test_hooks_selection_restore_and_loss_match(J):
    from paper_conf_eurosys_guptakkvgkrs24_b200.torch_hooks import attach, state_table
    shm = f"/dev/shm/jitc-hooks-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    torch.use_deterministic_algorithms(True, warn_only=True)
    g = torch.Generator(device="cuda").manual_seed(5)
    data = [(torch.randn(64, 256, device="cuda", generator=g), torch.randn(64, 256, device="cuda", generator=g))
            for _ in range(6)]
    reps, opts, ctxs, hooks = [], [], [], []
    try:
        for r in range(2):                                  # two DP replicas, same init, same data
            m = _model(1)
            o = torch.optim.Adam(m.parameters(), lr=1e-3)
            _step(m, o, *data[0])                           # creates the Adam state
            ctx = J.Context(device=0, rank=r, world=2, chunk_bytes=4096, image_dir=shm, staging_bytes=8 << 20,
                            slot_bytes=1 << 20)
            ctx.register(0, J.REQUIRED, [0, 1], state_table(m, o), keepalive=(m, o))
            hooks.append(attach(ctx, o, 0, version=1))
            reps.append(m), opts.append(o), ctxs.append(ctx)
        for x, y in data[1:3]:
            for m, o in zip(reps, opts):
                _step(m, o, x, y)
        torch.cuda.synchronize()
        assert ctxs[0].phase(0) == (3, J.CLEAN) and ctxs[1].phase(0) == (3, J.CLEAN)
        # replica 1 fails inside its optimizer step: the pre-hook ran, the post-hook never did
        x, y = data[3]
        opts[1].zero_grad(set_to_none=False)
        torch.nn.functional.mse_loss(reps[1](x), y).backward()
        ctxs[1].mark(0, hooks[1].version, J.DIRTY, torch.cuda.current_stream().cuda_stream)
        for p in list(reps[1].parameters())[:2]:            # ... and updated only part of its state
            p.data.add_(1e-3)
        torch.cuda.synchronize()
        blobs = ctxs[0].fingerprint() + ctxs[1].fingerprint()
        st, sel = J.select_consistent_replica(blobs, [0, 1])
        s = J.parse_selection(sel)
        assert st == J.OK and s["v_star"] == 3
        assert s["groups"][0]["writers"] == [0] and s["groups"][0]["excluded"] == [(1, J.DIRTY)]
        ctxs[0].capture(sel)
        import pickle
        cpu_state = {"version": 3, "adam_steps": [opts[0].state[p]["step"].item() for p in reps[0].parameters()],
                     "torch_rng": torch.get_rng_state()}
        ctxs[0].set_aux(pickle.dumps(cpu_state))             # the user's CPU state rides in the manifest
        ctxs[0].commit(sel)
        # a replacement for rank 1: fresh model + optimizer, restored from the image
        m2 = _model(99)
        o2 = torch.optim.Adam(m2.parameters(), lr=1e-3)
        _step(m2, o2, *data[5])
        ctx2 = J.Context(device=0, rank=1, world=2, chunk_bytes=4096, image_dir=shm, staging_bytes=8 << 20,
                         slot_bytes=1 << 20)
        ctx2.register(0, J.REQUIRED, [0, 1], state_table(m2, o2), keepalive=(m2, o2))
        ctx2.restore(0, J.HOST)
        ctx2.verify(0)
        torch.cuda.synchronize()
        for (n, a), b in zip(reps[0].state_dict().items(), m2.state_dict().values()):
            assert torch.equal(a, b), n
        restored_cpu = pickle.loads(ctx2.get_aux(0))
        assert restored_cpu["version"] == 3 and torch.equal(restored_cpu["torch_rng"], cpu_state["torch_rng"])
        for i, (p0, p2) in enumerate(zip(reps[0].parameters(), m2.parameters())):
            for k in ("exp_avg", "exp_avg_sq"):
                assert torch.equal(opts[0].state[p0][k], o2.state[p2][k])
            o2.state[p2]["step"].fill_(restored_cpu["adam_steps"][i])   # CPU scalar from the manifest's aux
        # training continues: the losses match bit for bit
        for x, y in data[3:]:
            la, lb = _step(reps[0], opts[0], x, y), _step(m2, o2, x, y)
            assert torch.equal(la, lb), (la.item(), lb.item())
        for h in hooks:
            h.remove()
        for c in ctxs + [ctx2]:
            c.close()
    finally:
        shutil.rmtree(shm, ignore_errors=True)
        torch.use_deterministic_algorithms(False)
