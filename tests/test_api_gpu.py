"""The paper's user API (Fig. 4) on a small bf16 model.

Ratel_init / Ratel_Optimizer / Ratel_hook on three MLP+LayerNorm blocks:
autograd accumulates into the wrapper's flat G16 buffers, post-accumulate
hooks hand each block off during backward, and after end_step() every
range's P32/m/v/P16 must equal the CPU oracle run on the same gradients.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icde_liaosyxcyww25_b200 as R
from paper_conf_icde_liaosyxcyww25_b200.api import Ratel_hook, Ratel_init, Ratel_Optimizer
from tests.tolerance import check_range

pytestmark = pytest.mark.gpu


class Block(torch.nn.Module):
    def __init__(self, d):
        super().__init__()
        self.fc1 = torch.nn.Linear(d, 4 * d)
        self.fc2 = torch.nn.Linear(4 * d, d)
        self.ln = torch.nn.LayerNorm(d)

    def forward(self, x):
        return x + self.fc2(torch.nn.functional.gelu(self.fc1(self.ln(x))))


@pytest.mark.parametrize("residency", ["device", "hybrid"])
def test_paper_api_matches_oracle(cuda_dev, residency):
    """residency="hybrid": the first 40 % of every range streamed through the
    GPU's tile ring, the rest updated by the CPU handler, one unit handed off
    as two library blocks -- both parts within R13 of the oracle."""
    torch.manual_seed(0)
    d, nb = 96, 3
    model = torch.nn.Sequential(*[Block(d) for _ in range(nb)]).to(cuda_dev)
    hp = dict(lr=2e-3, beta1=0.9, beta2=0.99, eps=1e-8, weight_decay=0.05)
    with Ratel_init():
        opt = Ratel_Optimizer([list(b.parameters()) for b in model], lr=hp["lr"],
                              betas=(hp["beta1"], hp["beta2"]), eps=hp["eps"],
                              weight_decay=hp["weight_decay"], residency=residency, hybrid_gpu_frac=0.4)
        if residency == "hybrid":
            assert all(len(v) == 2 for v in opt._lib_ids.values())
        Ratel_hook(opt)
        assert all(p.dtype == torch.bfloat16 for p in model.parameters())
        refs = []
        for bi in range(nb):
            for (master, m, v, p16, g16), rng in zip(opt.state(bi), opt.blocks[bi]):
                n = rng.numel
                refs.append((bi, rng, oracle.Range.fresh(master[:n].cpu().numpy(), int(rng.apply_wd))))
        x = torch.randn(64, d, device=cuda_dev, dtype=torch.bfloat16)
        launches0 = R.ratel_launch_count()
        for t in range(1, 5):
            opt.begin_step()
            loss = model(x).float().pow(2).mean()
            loss.backward()
            torch.cuda.synchronize()
            assert len(opt._handed) == nb           # every block handed off by its hooks
            grads = [r.g16[:r.numel].view(torch.int16).cpu().numpy().view(np.uint16) for _, r, _ in refs]
            opt.end_step()
            torch.cuda.synchronize()
            for (bi, rng, ref), g in zip(refs, grads):
                oracle.adam_range(ref, g, oracle.hparams(step=t, **hp))
                got = dict(p32=rng.master[:rng.numel].cpu().numpy(), m32=rng.m[:rng.numel].cpu().numpy(),
                           v32=rng.v[:rng.numel].cpu().numpy(),
                           p16=rng.p16[:rng.numel].view(torch.int16).cpu().numpy().view(np.uint16))
                check_range(got, ref, own_rne=oracle.bf16_rne, what=f"api step {t} block {bi}")
        if residency == "device":
            assert R.ratel_launch_count() - launches0 == 4 * nb
        opt.remove_hooks()
        del opt


def test_paper_api_state_dict_resume(cuda_dev):
    """Ratel_Optimizer.state_dict()/load_state_dict(): 3 steps, save, rebuild
    model + optimizer from the saved states, 2 more steps == 5 straight steps."""
    def build():
        torch.manual_seed(1)
        return torch.nn.Sequential(*[Block(64) for _ in range(2)]).to(cuda_dev)

    x = torch.randn(32, 64, device=cuda_dev, dtype=torch.bfloat16)

    def train(model, opt, n):
        for _ in range(n):
            opt.begin_step()
            model(x).float().pow(2).mean().backward()
            opt.end_step()
        torch.cuda.synchronize()

    def snap(opt):
        return [t.cpu().clone() for ranges in opt.blocks for r in ranges for t in (r.master, r.m, r.v, r.p16)]

    with Ratel_init():
        m1 = build()
        o1 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m1]))
        train(m1, o1, 5)
        want = snap(o1)
        o1.remove_hooks()
    with Ratel_init():
        m2 = build()
        o2 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m2]))
        train(m2, o2, 3)
        sd = o2.state_dict()
        o2.remove_hooks()
    with Ratel_init():
        m3 = build()
        o3 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m3]))
        o3.load_state_dict(sd)
        train(m3, o3, 2)
        got = snap(o3)
        o3.remove_hooks()
    for a, b in zip(want, got):
        assert torch.equal(a.view(torch.int16) if a.dtype == torch.bfloat16 else a.view(torch.int32),
                           b.view(torch.int16) if b.dtype == torch.bfloat16 else b.view(torch.int32))


@pytest.mark.parametrize("residency", ["device", "host"])
def test_paper_api_tensor_granularity_bitwise(cuda_dev, residency):
    """granularity="tensor" (one unit per weight matrix + one for the block's
    biases/norms, each handed off by its own hook as soon as its gradient is
    complete) updates every element exactly as block granularity does (R16):
    the model's bf16 parameters and fp32 masters agree bitwise after 4 steps,
    and every unit was handed off during backward."""
    def build():
        torch.manual_seed(2)
        return torch.nn.Sequential(*[Block(64) for _ in range(3)]).to(cuda_dev)

    x = torch.randn(48, 64, device=cuda_dev, dtype=torch.bfloat16)
    out = {}
    for gran in ("block", "tensor"):
        with Ratel_init():
            model = build()
            opt = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in model], residency=residency,
                                             granularity=gran))
            assert len(opt.block_ids) == (3 if gran == "block" else 3 * 3)   # fc1.w, fc2.w, {biases, ln}
            for _ in range(4):
                opt.begin_step()
                model(x).float().pow(2).mean().backward()
                assert len(opt._handed) == len(opt.block_ids)   # all units by hooks, during backward
                opt.end_step()
            torch.cuda.synchronize()
            out[gran] = ([p.detach().view(torch.int16).cpu().clone() for p in model.parameters()],
                         sorted(torch.cat([r.master.cpu() for rs in opt.blocks for r in rs]).view(torch.int32).tolist()))
            opt.remove_hooks()
    for a, b in zip(out["block"][0], out["tensor"][0]):
        assert torch.equal(a, b)
    assert out["block"][1] == out["tensor"][1]


def test_paper_api_ssd_residency_bitwise(cuda_dev, tmp_path):
    """residency="ssd": the wrapper writes theta0 into one state file, hands
    the library an O_DIRECT fd, and every step streams the states through the
    reader/writer threads -- same bits as device residency (R16), and
    state_dict() reads the file back; load_state_dict() into a fresh SSD
    optimizer then continues bitwise like an uninterrupted run."""
    def build():
        torch.manual_seed(3)
        return torch.nn.Sequential(*[Block(64) for _ in range(2)]).to(cuda_dev)

    x = torch.randn(32, 64, device=cuda_dev, dtype=torch.bfloat16)

    def train(model, opt, n):
        for _ in range(n):
            opt.begin_step()
            model(x).float().pow(2).mean().backward()
            opt.end_step()
        torch.cuda.synchronize()

    def snap(model, opt):
        sd = opt.state_dict()
        return ([p.detach().view(torch.int16).cpu().clone() for p in model.parameters()],
                [t.view(torch.int32) for rs in sd["ranges"] for r in rs for t in r.values()])

    cfg = dict(tile_elems=4096)
    with Ratel_init(**cfg):
        m0 = build()
        o0 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m0]))
        train(m0, o0, 5)
        want = snap(m0, o0)
        o0.remove_hooks()
    with Ratel_init(**cfg):
        m1 = build()
        o1 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m1], residency="ssd",
                                        ssd_path=str(tmp_path / "a.bin")))
        train(m1, o1, 3)
        sd = o1.state_dict()
        o1.remove_hooks()
    o1.close()
    with Ratel_init(**cfg):
        m2 = build()
        o2 = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in m2], residency="ssd",
                                        ssd_path=str(tmp_path / "b.bin")))
        o2.load_state_dict(sd)
        train(m2, o2, 2)
        got = snap(m2, o2)
        o2.remove_hooks()
    o2.close()
    for a, b in zip(want[0], got[0]):
        assert torch.equal(a, b)
    for a, b in zip(want[1], got[1]):
        assert torch.equal(a, b)


def test_paper_api_ssd_hostcompute_equals_hostcompute(cuda_dev, tmp_path):
    """residency="ssd_hostcompute" (states in one state file, the CPU handler on
    each staged tile -- the paper's full pipeline) gives the same bits as the
    CPU handler on pinned states, through the paper's API, for 3 steps."""
    def build():
        torch.manual_seed(4)
        return torch.nn.Sequential(*[Block(64) for _ in range(2)]).to(cuda_dev)

    x = torch.randn(32, 64, device=cuda_dev, dtype=torch.bfloat16)
    out = []
    for residency, kw in (("hostcompute", {}), ("ssd_hostcompute", {"ssd_path": str(tmp_path / "s.bin")})):
        with Ratel_init(tile_elems=4096, host_threads=4):
            model = build()
            opt = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in model], residency=residency, **kw))
            for _ in range(3):
                opt.begin_step()
                model(x).float().pow(2).mean().backward()
                opt.end_step()
            torch.cuda.synchronize()
            sd = opt.state_dict()
            out.append(([p.detach().view(torch.int16).cpu().clone() for p in model.parameters()],
                        [t.view(torch.int32) for rs in sd["ranges"] for r in rs for t in r.values()]))
            opt.remove_hooks()
        opt.close()
    for a, b in zip(out[0][0], out[1][0]):
        assert torch.equal(a, b)
    for a, b in zip(out[0][1], out[1][1]):
        assert torch.equal(a, b)


def test_paper_api_gradient_accumulation_matches_oracle(cuda_dev):
    """begin_step(micro_batches=2): autograd accumulates two backward passes
    into the flat G16 buffers; every unit is handed off during the second
    one (not the first), and the update equals the oracle on the accumulated
    gradient."""
    torch.manual_seed(5)
    d, nb = 64, 2
    model = torch.nn.Sequential(*[Block(d) for _ in range(nb)]).to(cuda_dev)
    hp = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=0.01)
    xs = [torch.randn(16, d, device=cuda_dev, dtype=torch.bfloat16) for _ in range(2)]
    with Ratel_init():
        opt = Ratel_hook(Ratel_Optimizer([list(b.parameters()) for b in model], lr=hp["lr"],
                                         weight_decay=hp["weight_decay"]))
        refs = []
        for bi in range(nb):
            for (master, m, v, p16, g16), rng in zip(opt.state(bi), opt.blocks[bi]):
                refs.append((rng, oracle.Range.fresh(master[:rng.numel].cpu().numpy(), int(rng.apply_wd))))
        for t in (1, 2):
            opt.begin_step(micro_batches=2)
            model(xs[0]).float().pow(2).mean().backward()
            torch.cuda.synchronize()
            assert len(opt._handed) == 0                 # nothing handed off after the first micro-batch
            model(xs[1]).float().pow(2).mean().backward()
            torch.cuda.synchronize()
            assert len(opt._handed) == nb
            grads = [r.g16[:r.numel].view(torch.int16).cpu().numpy().view(np.uint16) for r, _ in refs]
            opt.end_step()
            torch.cuda.synchronize()
            for (rng, ref), g in zip(refs, grads):
                oracle.adam_range(ref, g, oracle.hparams(step=t, **hp))
                got = dict(p32=rng.master[:rng.numel].cpu().numpy(), m32=rng.m[:rng.numel].cpu().numpy(),
                           v32=rng.v[:rng.numel].cpu().numpy(),
                           p16=rng.p16[:rng.numel].view(torch.int16).cpu().numpy().view(np.uint16))
                check_range(got, ref, own_rne=oracle.bf16_rne, what=f"accumulation step {t}")
        opt.remove_hooks()
