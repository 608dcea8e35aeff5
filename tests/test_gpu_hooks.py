"""the activation detector finds the first module whose output
holds NaN / INF (the SRU uninitialised-tensor case, recast for
model code), through fpx_scan_tensor forward hooks."""
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.mark.parametrize("batch", [False, True], ids=["per-output", "one-launch"])
def test_activation_scanner_finds_first_nan_module(batch):
    from paper_conf_hpdc_lilfslg23_b200.hooks import ActivationScanner
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    torch.manual_seed(0)
    model = torch.nn.Sequential(
        torch.nn.Linear(64, 128), torch.nn.ReLU(), torch.nn.Linear(128, 128), torch.nn.Tanh(),
        torch.nn.Linear(128, 10),
    ).cuda()
    x = torch.randn(32, 64, device="cuda")
    sc = ActivationScanner(model, batch=batch)
    model(x)
    assert sc.first_exception() is None  # clean forward
    with torch.no_grad():
        model[2].weight[5, 7] = float("nan")  # poison the second Linear
    model(x)
    model(x)
    call, name, element, kind = sc.first_exception()
    assert (call, name, kind) == (2, "2", fpx.NAN)
    assert element % 128 == 5  # output column 5 of the first row that reaches it
    ents = sc.entries()
    sites = {sc.names[int(e["site"])] for e in ents}
    assert sites == {"2", "3", "4"}  # NaN propagates to every later layer
    sc.remove()


def test_activation_scanner_with_selective_policy():
    from paper_conf_hpdc_lilfslg23_b200.hooks import ActivationScanner, SelectivePolicy

    model = torch.nn.Sequential(torch.nn.Linear(16, 16), torch.nn.Linear(16, 16)).cuda()
    with torch.no_grad():
        model[0].weight[0, 0] = float("inf")
    x = torch.ones(4, 16, device="cuda")
    sc = ActivationScanner(model, policy=SelectivePolicy(white_list={"1"}, k=2))
    for _ in range(4):
        model(x)
    ents = sc.entries()
    # only module "1" is scanned, on forward calls 1 and 3 (1 in 2)
    assert {sc.names[int(e["site"])] for e in ents} == {"1"}
    assert len(sc.seq) == 2 and [c for c, _ in sc.seq] == [1, 3]
    sc.remove()


@pytest.mark.parametrize("batch", [False, True], ids=["per-output", "one-launch"])
def test_activation_scanner_entries_match_oracle(batch):
    """Every hooked output, copied to the host and scanned by the oracle at the
    same site and base index (seq << 36), gives the scanner's table entry by
    entry (not only the first-exception attribution)."""
    import numpy as np

    import oracle
    from _records import describe_diff, entries_equal
    from paper_conf_hpdc_lilfslg23_b200.hooks import SEQ_SHIFT, ActivationScanner

    torch.manual_seed(1)
    model = torch.nn.Sequential(
        torch.nn.Linear(64, 96), torch.nn.GELU(), torch.nn.Linear(96, 96), torch.nn.LayerNorm(96),
        torch.nn.Linear(96, 32),
    ).cuda()
    with torch.no_grad():
        model[0].weight[3, 0] = float("inf")    # column 3 of the first output: +-INF (NaN where x = 0 / NaN)
        model[2].bias[7] = 1e-41                 # a subnormal bias: subnormals in later outputs
    x = torch.randn(16, 64, device="cuda")
    x[2, 5] = float("nan")                       # row 2: NaN everywhere downstream
    sc = ActivationScanner(model, batch=batch)
    captured = []
    caps = [m.register_forward_hook(lambda m_, a, out: captured.append(out.detach().clone()))
            for name, m in model.named_modules() if not any(True for _ in m.children())]
    for _ in range(3):
        model(x)
    got = sc.entries()
    assert len(captured) == len(sc.seq) == 15
    ref = oracle.Table()
    for i, t in enumerate(captured):
        _, site = sc.seq[i]
        host = t.contiguous().view(torch.int32).cpu().numpy()
        ref.scan_tensor(host, 0, site=site, base_index=i << SEQ_SHIFT)
    exp = ref.entries()
    assert entries_equal(got, exp), describe_diff(got, exp)
    assert {int(k) for k in exp["kind"]} >= {0, 1}
    for c in caps:
        c.remove()
    sc.remove()
