"""GPU parity of pm_histogram_match (Sec. II; reading R12) with the
oracle's histogram matching: bit-exact u8 images on every shape, family and
channel count, in place and out of place, at the BASELINE sizes."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


@pytest.mark.parametrize("fam", ["smooth", "noise", "ties", "identical", "shuffle"])
@pytest.mark.parametrize("N,M,C", [(128, 8, 3), (512, 16, 3), (90, 10, 3), (200, 5, 1), (33, 11, 3), (7, 7, 1)])
def test_histogram_match_parity(fam, N, M, C):
    I, T = synth.make_pair(fam, N, M, C, seed=N)
    got = pm.histogram_match(dev(I), dev(T)).cpu().numpy()
    assert (got == oracle.histogram_match(I, T)).all()


def test_histogram_match_in_place_and_2d():
    I, T = synth.make_pair("smooth", 512, 16, 3, seed=1)
    dI = dev(I)
    pm.histogram_match(dI, dev(T), out=dI)
    assert (dI.cpu().numpy() == oracle.histogram_match(I, T)).all()
    g, h = I[:, :, 0].copy(), T[:, :, 1].copy()
    assert (pm.histogram_match(dev(g), dev(h)).cpu().numpy() == oracle.histogram_match(g, h)).all()


def test_histogram_match_unaligned_buffers():
    # image pointers off 16-byte alignment: the byte-wise path, same result
    I, T = synth.make_pair("noise", 64, 8, 3, seed=2)
    bi = torch.empty(I.size + 16, dtype=torch.uint8, device=DEV)
    bt = torch.empty(T.size + 16, dtype=torch.uint8, device=DEV)
    dI = bi[3:3 + I.size].view(64, 64, 3)
    dT = bt[5:5 + T.size].view(64, 64, 3)
    dI.copy_(dev(I))
    dT.copy_(dev(T))
    assert (pm.histogram_match(dI, dT).cpu().numpy() == oracle.histogram_match(I, T)).all()


@pytest.mark.parametrize("cfg", [4, 5])
def test_histogram_match_full_size(cfg):
    I, T = synth.config_pair(cfg, "smooth", 0)
    assert (pm.histogram_match(dev(I), dev(T)).cpu().numpy() == oracle.histogram_match(I, T)).all()


def test_histogram_match_then_photomosaic():
    # the paper's pipeline order (P:84 then Steps 1-3): adjusted input -> E -> Alg. 2
    I, T = synth.make_pair("smooth", 512, 16, 3, seed=3)
    Ih = oracle.histogram_match(I, T)
    E_ref = oracle.error_matrix(Ih, T, 16)
    ref = oracle.local_search(E_ref)
    dI = pm.histogram_match(dev(I), dev(T))
    perm, rounds, swaps, c, E = pm.photomosaic(dI, dev(T), 16)
    assert (E.cpu().numpy() == E_ref).all()
    assert (perm.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])


def test_histogram_match_invalid():
    L = pm.lib()
    x = torch.zeros((8, 8, 3), dtype=torch.uint8, device=DEV)
    y = torch.zeros((8, 8, 3), dtype=torch.uint8, device=DEV)
    assert L.pm_histogram_match(x.data_ptr(), y.data_ptr(), 8, 3, y.data_ptr(), None) == pm.PM_ERR_INVALID
    assert L.pm_histogram_match(None, y.data_ptr(), 8, 3, x.data_ptr(), None) == pm.PM_ERR_INVALID
    assert L.pm_histogram_match(x.data_ptr(), y.data_ptr(), 2, 5, x.data_ptr(), None) == pm.PM_ERR_UNSUPPORTED
