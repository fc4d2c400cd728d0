"""GPU parity for the bezier-surface loop (Listing 2; SURVEY.md §8f NEXT 4;
DESIGN.md §6.9): every variant of csrc/bezier.cu through the C ABI against the CPU oracle
(oracle/bezier_oracle.c).  All variants execute the same floating-point operations in the
same order, so the bar is bit-exact in fp64 and in fp32."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from xs_workloads import BEZIER_SEED, BEZIER_WORKLOADS, bezier_control_net  # noqa: E402

VARIANTS = ["M", "M2", "U1", "U2", "S", "T"]
DTYPES = [(torch.float64, np.float64), (torch.float32, np.float32)]


@pytest.fixture(scope="module")
def xs():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_cgo_murtovigplls24_b200 as pkg
    return pkg


def _bits_equal(a: np.ndarray, b: np.ndarray) -> bool:
    return a.shape == b.shape and a.dtype == b.dtype and np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("tdt,ndt", DTYPES)
def test_blend_loop_every_k_n(xs, oracle_mod, variant, tdt, ndt):
    # the bare loop for every 0 <= k <= n <= 64 (divergent per lane by construction)
    ks, ns = zip(*[(k, n) for n in range(65) for k in range(n + 1)])
    k = torch.tensor(ks, dtype=torch.int32, device="cuda")
    n = torch.tensor(ns, dtype=torch.int32, device="cuda")
    got = xs.bezier_blend(k, n, None, variant=variant, dtype=tdt).cpu().numpy()
    ref = np.array([oracle_mod.blend_loop(a, b, ndt) for a, b in zip(ks, ns)], dtype=ndt)
    assert _bits_equal(got, ref)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("tdt,ndt", DTYPES)
def test_bezier_blend_with_powers(xs, oracle_mod, variant, tdt, ndt):
    rng = np.random.default_rng(BEZIER_SEED)
    ns = rng.integers(0, 33, 3000)
    ks = np.array([rng.integers(0, v + 1) for v in ns])
    mus = rng.random(3000).astype(ndt)
    mus[:4] = [0.0, 1.0, 0.5, 1e-3]
    got = xs.bezier_blend(torch.tensor(ks, device="cuda"), torch.tensor(ns, device="cuda"),
                          torch.tensor(mus, device="cuda"), variant=variant, dtype=tdt).cpu().numpy()
    ref = np.array([oracle_mod.bezier_blend(int(a), float(m), int(b), ndt) for a, m, b in zip(ks, mus, ns)], dtype=ndt)
    assert _bits_equal(got, ref)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("tdt,ndt", DTYPES)
def test_surface_tiny(xs, oracle_mod, variant, tdt, ndt):
    w = BEZIER_WORKLOADS["tiny"]
    P = bezier_control_net(w.ni, w.nj, dtype=ndt)
    ref = oracle_mod.bezier_surface(P, w.res_i, w.res_j)
    got = xs.bezier_surface(torch.tensor(P, device="cuda"), w.res_i, w.res_j, variant=variant).cpu().numpy()
    assert _bits_equal(got, ref)


@pytest.mark.parametrize("ni,nj,ri,rj", [(0, 0, 2, 2), (0, 3, 5, 17), (3, 0, 17, 5), (1, 1, 2, 33),
                                         (32, 32, 19, 21), (7, 31, 16, 16), (2, 9, 33, 47), (5, 4, 2, 2)])
@pytest.mark.parametrize("variant", VARIANTS)
def test_surface_edge_nets(xs, oracle_mod, ni, nj, ri, rj, variant):
    for tdt, ndt in DTYPES:
        P = bezier_control_net(ni, nj, seed=ni * 100 + nj, dtype=ndt)
        ref = oracle_mod.bezier_surface(P, ri, rj)
        got = xs.bezier_surface(torch.tensor(P, device="cuda"), ri, rj, variant=variant).cpu().numpy()
        assert _bits_equal(got, ref), (ni, nj, ri, rj, variant, ndt)


@pytest.mark.parametrize("name", ["paper", "deep"])
@pytest.mark.parametrize("tdt,ndt", DTYPES)
def test_surface_full_size_sampled(xs, oracle_mod, name, tdt, ndt):
    # BASELINE-sized surfaces in the launch configuration the A/B times: every variant
    # equal to T on the whole surface, T equal to the oracle on sampled points + corners
    w = BEZIER_WORKLOADS[name]
    P = bezier_control_net(w.ni, w.nj, dtype=ndt)
    Pt = torch.tensor(P, device="cuda")
    ref_t = xs.bezier_surface(Pt, w.res_i, w.res_j, variant="T")
    for v in VARIANTS[:-1]:
        assert torch.equal(xs.bezier_surface(Pt, w.res_i, w.res_j, variant=v), ref_t), v
    rng = np.random.default_rng(1)
    ii = np.concatenate([[0, 0, w.res_i - 1, w.res_i - 1], rng.integers(0, w.res_i, 1500)])
    jj = np.concatenate([[0, w.res_j - 1, 0, w.res_j - 1], rng.integers(0, w.res_j, 1500)])
    ref = oracle_mod.bezier_surface_points(P, w.res_i, w.res_j, ii, jj)
    got = ref_t.cpu().numpy()[ii, jj]
    assert _bits_equal(got, ref)


def test_stream_and_out_buffer(xs, oracle_mod):
    w = BEZIER_WORKLOADS["tiny"]
    P = bezier_control_net(w.ni, w.nj)
    s = torch.cuda.Stream()
    out = torch.full((w.res_i, w.res_j, 3), float("nan"), dtype=torch.float64, device="cuda")
    with torch.cuda.stream(s):
        xs.bezier_surface(torch.tensor(P, device="cuda"), w.res_i, w.res_j, variant="U2", out=out, stream=s)
    s.synchronize()
    assert _bits_equal(out.cpu().numpy(), oracle_mod.bezier_surface(P, w.res_i, w.res_j))


def test_validation(xs):
    P = torch.zeros((6, 5, 3), dtype=torch.float64, device="cuda")
    out = torch.empty((8, 8, 3), dtype=torch.float64, device="cuda")
    bad = [
        (33, 4, 8, 8, xs.XS_F64, 0, P, out),   # ni > 32
        (5, 4, 1, 8, xs.XS_F64, 0, P, out),    # res < 2
        (5, 4, 8, 8, 7, 0, P, out),            # dtype
        (5, 4, 8, 8, xs.XS_F64, 6, P, out),    # variant
        (5, 4, 8, 8, xs.XS_F64, 0, None, out), # ctrl
        (5, 4, 1 << 21, 1 << 20, xs.XS_F64, 0, P, out),  # res_i * res_j >= 2^40
    ]
    for args in bad:
        with pytest.raises(xs.XSError) as e:
            xs.xs_bezier_surface(*args)
        assert e.value.code == xs.XS_EINVAL
    with pytest.raises(xs.XSError):
        xs.xs_bezier_blend(4, None, None, None, xs.XS_F64, 0, None)
    xs.xs_bezier_blend(0, None, None, None, xs.XS_F64, 0, None)   # empty is fine
