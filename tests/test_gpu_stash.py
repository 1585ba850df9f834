"""f2: stash-time encodings inside PyTorch autograd (paper_conf_isca_jainpmtp18_b200.stash).
The Binarize and SSDC paths are lossless, so a training step's gradients match
plain PyTorch up to the dense-layer backward's own rounding; DPR is lossy and stays
within its format's relative error."""
import pytest
import torch
import torch.nn as nn
import torch.nn.functional as F

pytestmark = pytest.mark.gpu


class TinyVGG(nn.Module):
    def __init__(self):
        super().__init__()
        self.c1, self.c2 = nn.Conv2d(3, 16, 3, padding=1), nn.Conv2d(16, 16, 3, padding=1)
        self.c3, self.c4 = nn.Conv2d(16, 32, 3, padding=1), nn.Conv2d(32, 32, 3, padding=1)
        self.fc = nn.Linear(32 * 8 * 8, 10)

    def base(self, x):
        x = F.max_pool2d(F.relu(self.c2(F.relu(self.c1(x)))), 2)
        x = F.max_pool2d(F.relu(self.c4(F.relu(self.c3(x)))), 2)
        return self.fc(torch.flatten(x, 1))

    def gist(self, x, stash):
        z = stash.relu_conv(self.c1(x), self.c2)
        z = stash.relu_maxpool(z, 2)
        z = stash.relu_conv(stash.stashed_conv(z, self.c3), self.c4)
        z = stash.relu_maxpool(z, 2)
        return self.fc(torch.flatten(z, 1))


def grads(model, fwd, x, y):
    model.zero_grad(set_to_none=True)
    F.cross_entropy(fwd(x), y).backward()
    return [p.grad.clone() for p in model.parameters()]


@pytest.fixture
def deterministic():
    """cuDNN picks the same deterministic algorithm for the same op and shapes, so a lossless stash
    must reproduce plain PyTorch's gradients bit for bit."""
    old = (torch.backends.cudnn.deterministic, torch.backends.cudnn.benchmark)
    torch.backends.cudnn.deterministic, torch.backends.cudnn.benchmark = True, False
    yield
    torch.backends.cudnn.deterministic, torch.backends.cudnn.benchmark = old


def test_lossless_stash_matches_pytorch_bit_exact(gist, cuda, deterministic):
    """Binarize and SSDC are lossless: the training step's gradients are identical to
    plain PyTorch's (north star: gradients recomputed from the encodings match bit-exactly)."""
    from paper_conf_isca_jainpmtp18_b200 import stash
    torch.manual_seed(0)
    m = TinyVGG().to(cuda)
    x = torch.randn(8, 3, 32, 32, device=cuda)
    y = torch.randint(0, 10, (8,), device=cuda)
    g0 = grads(m, m.base, x, y)
    g0b = grads(m, m.base, x, y)
    assert all(torch.equal(a, b) for a, b in zip(g0, g0b)), "plain PyTorch itself is not reproducible"
    g1 = grads(m, lambda t: m.gist(t, stash), x, y)
    for (name, _), a, b in zip(m.named_parameters(), g0, g1):
        assert torch.equal(a.view(torch.int32), b.view(torch.int32)), name


def test_dpr_saved_tensors_hooks(gist, cuda):
    from paper_conf_isca_jainpmtp18_b200 import stash
    torch.manual_seed(1)
    lin = nn.Linear(4096, 256).to(cuda)
    x = torch.randn(64, 4096, device=cuda, requires_grad=True)
    out0 = lin(x)
    out0.sum().backward()
    gw0 = lin.weight.grad.clone()
    lin.weight.grad = None
    with stash.dpr_saved_tensors(16, lin.parameters()):
        out1 = lin(x)
    out1.sum().backward()
    # the saved input went through FP16: weight grad within fp16 relative error
    torch.testing.assert_close(lin.weight.grad, gw0, rtol=2e-3, atol=2e-2)
    assert not torch.equal(lin.weight.grad, gw0)  # the stash really was reduced


def test_csr_stash_is_exact_and_small(gist, cuda):
    from paper_conf_isca_jainpmtp18_b200 import stash
    y = torch.relu(torch.randn(4, 64, 56, 56, device=cuda) - 0.84)  # ~80% zeros
    s = stash.CSRStash(y)
    assert torch.equal(s.dense().view(torch.int32), y.view(torch.int32))
    assert s.nbytes() < 0.3 * 4 * y.numel()


def test_arena_stash_one_pass_no_sync_bit_exact(gist, cuda, deterministic):
    """f2 single pass: inside ssdc_arena every stash is ONE encode into a chained arena with
    device-side offsets.  The forward runs under torch's sync debug mode set to "error" (any host
    synchronization raises), and the gradients still equal plain PyTorch's bit for bit."""
    from paper_conf_isca_jainpmtp18_b200 import stash
    torch.manual_seed(0)
    m = TinyVGG().to(cuda)
    x = torch.randn(8, 3, 32, 32, device=cuda)
    y = torch.randint(0, 10, (8,), device=cuda)
    g0 = grads(m, m.base, x, y)
    arena = stash.StashArena(8 * 16 * 32 * 32 * 4, cuda)  # >= every SSDC-stashed element of the step
    launches0 = gist.gist_launch_count()
    m.zero_grad(set_to_none=True)
    torch.cuda.synchronize()
    with stash.ssdc_arena(arena):
        torch.cuda.set_sync_debug_mode("error")
        try:
            logits = m.gist(x, stash)
        finally:
            torch.cuda.set_sync_debug_mode("default")
    assert gist.gist_launch_count() - launches0 >= 3  # the three SSDC stashes were encoded
    F.cross_entropy(logits, y).backward()
    g1 = [p.grad.clone() for p in m.parameters()]
    for (name, _), a, b in zip(m.named_parameters(), g0, g1):
        assert torch.equal(a.view(torch.int32), b.view(torch.int32)), name
    used = arena.check()
    # the arena holds exactly the nonzeros of the three stashed maps
    assert 0 < used <= arena.capacity


def test_arena_overflow_is_reported_before_decode(gist, cuda):
    from paper_conf_isca_jainpmtp18_b200 import stash
    y = torch.relu(torch.randn(2, 16, 32, 32, device=cuda))
    arena = stash.StashArena(100, cuda)  # far too small
    with stash.ssdc_arena(arena):
        s = stash.CSRStash(y)
    with pytest.raises(stash.StashOverflow) as e:
        s.dense()
    assert e.value.needed == int((y.view(torch.int32) != 0).sum().item())
    # a fresh arena large enough round-trips exactly, and reset() reuses it
    arena = stash.StashArena(y.numel(), cuda)
    for _ in range(2):
        arena.reset()
        with stash.ssdc_arena(arena):
            s = stash.CSRStash(y)
            s2 = stash.CSRStash(2 * y)
        assert torch.equal(s.dense().view(torch.int32), y.view(torch.int32))
        assert torch.equal(s2.dense().view(torch.int32), (2 * y).view(torch.int32))


def test_arena_plan_per_group_resizes_and_stays_exact(gist, cuda, deterministic):
    """ArenaPlan: one arena per group, sized from the previous step.  A first step with a too-small
    capacity raises StashOverflow at the first decode; update() reads every group's end in one
    synchronization, and the redone step is bit-exact to plain PyTorch."""
    from paper_conf_isca_jainpmtp18_b200 import stash
    torch.manual_seed(0)
    m = TinyVGG().to(cuda)
    x = torch.randn(8, 3, 32, 32, device=cuda)
    y = torch.randint(0, 10, (8,), device=cuda)
    g0 = grads(m, m.base, x, y)
    plan = stash.ArenaPlan(cuda, floor=16)

    def fwd(t):
        with stash.ssdc_arena(plan.arena("a", 64)):
            z = stash.relu_conv(m.c1(t), m.c2)
        z = stash.relu_maxpool(z, 2)
        with stash.ssdc_arena(plan.arena("b", 64)):
            z = stash.relu_conv(stash.stashed_conv(z, m.c3), m.c4)
        z = stash.relu_maxpool(z, 2)
        return m.fc(torch.flatten(z, 1))

    with pytest.raises(stash.StashOverflow):
        grads(m, fwd, x, y)
    sizes = plan.update()
    assert set(sizes) == {"a", "b"} and all(used > cap for used, cap in sizes.values())
    g1 = grads(m, fwd, x, y)
    after = plan.update()
    assert all(used <= cap for used, cap in after.values())
    for (name, _), a, b in zip(m.named_parameters(), g0, g1):
        assert torch.equal(a.view(torch.int32), b.view(torch.int32)), name
