"""CPU-side checks of the product library (no GPU needed, no kernel launches):
the C ABI loads and exports every symbol include/cswap.h declares, and the pure-host
parts (selector, LR/link fits, size bounds) agree with the oracle / numpy."""
import itertools
import os
import re

import numpy as np
import pytest

import synth
from oracle import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def C():
    from paper_conf_cluster_chenhzchysc21_b200 import build
    build.build()
    from paper_conf_cluster_chenhzchysc21_b200 import cswap
    return cswap


def header_symbols():
    src = open(os.path.join(ROOT, "include", "cswap.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cswap_[a-z_0-9]+)\s*\(", src)))


def test_every_declared_symbol_is_exported(C):
    import ctypes
    lib = ctypes.CDLL(C.LIB_PATH)
    syms = header_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(lib, s), f"{s} declared in include/cswap.h but not exported"
    assert set(syms) == set(C.EXPORTED), "binding and header disagree"


def test_not_initialised_reports_status(C):
    with pytest.raises(C.CswapError) as e:
        C.compress(0, 10, C.F32, C.ZVC, 0, 0, 0)
    assert e.value.status == 7  # NOT_READY


def to_product_calib(C, oc):
    c = C.Calib()
    for f, _ in C.Calib._fields_:
        if f in ("reserved",):
            continue
        src = "pad_" if f == "reserved" else f
        v = getattr(oc, src)
        if f == "beta":
            for i in range(len(v)):
                c.beta[i] = v[i]
        else:
            setattr(c, f, v)
    return c


def test_selector_matches_oracle_grid(C):
    rng = np.random.default_rng(11)
    beta = rng.uniform(0, 2e-12, size=(4, 2, 6, 3))
    beta[..., 0] = rng.uniform(1e-6, 3e-5, size=(4, 2, 6))
    tensors = {
        "iid": lambda n, s: synth.relu_iid(n, s, seed=n),
        "clu": lambda n, s: synth.relu_clustered(n, min(max(s, .05), .95), 40, seed=n + 1),
        "zero": lambda n, s: np.zeros(n, np.uint32),
    }
    checked = 0
    for (kind, gen), n, s, mode, F, bw, hf in itertools.product(
            tensors.items(), [1, 1000, 70000, 300000], [0.0, 0.3, 0.6, 0.95], [0, 1], [1024, 1 << 22],
            [8e9, 55e9], [0.0, 2e-5]):
        x = gen(n, s)
        counts = O.probe(x, O.F32)
        oc = O.make_calib(alpha_d2h=8e-6, bw_d2h=bw, alpha_h2d=9e-6, bw_h2d=bw * 0.9, beta=beta, mode=mode,
                          frame_elems=F, lz4_gamma1=3.0, lz4_gamma2=1.0, margin=0.05)
        ref = O.select(n, O.F32, counts, hf, hf / 2, oc)
        got = C.select_from_probe(n, C.F32, counts, hf, hf / 2, to_product_calib(C, oc)).as_dict()
        assert got["codec"] == ref["codec"]
        for key in ("t_pred", "t_prime"):
            assert got[key] == ref[key]
        assert got["t_codec"] == ref["t_codec"] and got["size"] == ref["size"]
        checked += 1
    assert checked > 500


def test_fit_time_model_matches_numpy(C):
    rng = np.random.default_rng(5)
    S = rng.uniform(20 * 2**20, 2000 * 2**20, 300)
    s = rng.uniform(0.2, 0.8, 300)
    t = 2e-5 + 3e-13 * S - 1e-13 * S * s + rng.normal(0, 1e-6, 300)
    got = np.array(C.fit_time_model(S, s, t))
    ref = O.lstsq_fit(S, s, t)
    assert np.allclose(got, ref, rtol=1e-7, atol=1e-12)
    exact = 4e-6 + 2.5e-13 * S + 7e-14 * S * s
    assert np.allclose(C.fit_time_model(S, s, exact), [4e-6, 2.5e-13, 7e-14], rtol=1e-7)


def test_fit_link(C):
    b = np.array([2**k for k in range(16, 31)], dtype=np.float64)
    t = 7e-6 + b / 52e9
    a, bw = C.fit_link(b, t)
    assert a == pytest.approx(7e-6, rel=1e-6) and bw == pytest.approx(52e9, rel=1e-9)


@pytest.mark.parametrize("codec", [0, 1, 2, 3, 4])
@pytest.mark.parametrize("dtype", [0, 1])
def test_max_size_matches_oracle(C, codec, dtype):
    for n in (0, 1, 1000, 5000, 70001):
        for F in (1024, 4096):
            param = {3: 512, 4: 2048}.get(codec, 0)
            fmt = (F, 512, 2048)
            assert C.max_compressed_size(n, dtype, codec, fmt) == O.max_size(codec, dtype, n, F, param)


def test_swap_target_needs_init(C):
    """cswap_set_swap_target (NEXT-4b) reports NOT_READY before cswap_init, like every call."""
    with pytest.raises(C.CswapError) as e:
        C.set_swap_target(1)
    assert e.value.status == 7
    with pytest.raises(C.CswapError) as e:
        C.get_swap_target()
    assert e.value.status == 7
