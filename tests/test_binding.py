"""Python binding validation (GPU): every tensor's shape / element count is checked against
the sizes passed to the C ABI before anything is launched (the ABI takes only N, p and
extents, so a short buffer would otherwise be an out-of-bounds device access)."""
import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bc():
    import paper_conf_icpp_nelsonrbhhjn15_b200 as m
    return m


def z(*shape):
    return torch.zeros(shape, dtype=torch.float64, device="cuda")


def test_spectral_shapes(bc):
    P1 = 5
    A, U = z(P1, P1), z(3, P1, P1, P1)
    with pytest.raises(ValueError):
        bc.sumfact3d(A, z(P1 + 1, P1 + 1), A, U)          # B not (p+1)x(p+1)
    with pytest.raises(ValueError):
        bc.sumfact3d(A, A, A, U, out=z(2, P1, P1, P1))    # short output
    with pytest.raises(ValueError):
        bc.sumfact3d(A, A, A, U, check_ws=z(100))         # short workspace
    with pytest.raises(ValueError):
        bc.sumfact2d(A, A, z(3, P1, P1), out=z(3, P1, P1 - 1))
    with pytest.raises(ValueError):
        bc.local_grad3(A, U, out=(z(3, P1, P1, P1), z(3, P1, P1, P1), z(2, P1, P1, P1)))
    with pytest.raises(ValueError):
        bc.local_grad3_t(A, U, U, z(2, P1, P1, P1))
    with pytest.raises(TypeError):
        bc.sumfact3d(A, A, A, U.float())


def test_ccsdt_sizes(bc):
    ext = (4, 4, 4, 3, 3, 3, 5)
    n3 = 4 ** 3 * 3 ** 3
    na, nb = bc.operand_sizes("d1", ext)
    t3, t2, v2 = z(n3), z(na), z(nb)
    bc.ccsdt("d1", 1, ext, t3, t2, v2)
    with pytest.raises(ValueError):
        bc.ccsdt("d1", 1, ext, z(n3 - 1), t2, v2)
    with pytest.raises(ValueError):
        bc.ccsdt("d1", 1, ext, t3, z(na - 1), v2)
    with pytest.raises(ValueError):
        bc.ccsdt_fused("d1", ext, t3, [t2] * 9, [v2] * 8 + [z(3)])
    with pytest.raises(ValueError):
        bc.ccsdt_fused("d1", ext, t3, [t2] * 9, [v2] * 8 + [None])
    with pytest.raises(ValueError):
        bc.check_energy(ext, t3, z(11), z(9))            # eps_h needs h1+h2+h3 = 12
    with pytest.raises(ValueError):
        bc.check_sumsq(t3, ws=z(10))
    torch.cuda.synchronize()
