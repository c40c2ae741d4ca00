"""Ghost-validity under poison: the ghost-shell parity tests again with every ghost cell of every field
starting as NaN (MG_POISON_GHOSTS=1, api.cu poison_ghosts; x's ghosts again after
mg_set_solution(NULL)).

The exchange refreshes only the ghost cells within its depth of the owned box (the
depth-limited exchange) and the schedule sweeps ghost bricks only as deep as they are valid (reading
A11).  Any kernel reading a ghost cell the exchange did not refresh -- beyond the exchange depth, or
stale since the last exchange -- would turn owned results into NaN, so these bitwise checks against
the oracle prove the validity bookkeeping for every transport, CA period, kernel family, boundary
condition, coefficient variant, brick edge and decomposition they cover.
"""
import pytest

import test_gpu_parity as P
import test_gpu_variants as V

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]


@pytest.fixture(autouse=True)
def _poison(monkeypatch):
    monkeypatch.setenv("MG_POISON_GHOSTS", "1")


@pytest.mark.parametrize("transport", [2, 1, 3])
@pytest.mark.parametrize("period", [0, 1, 2, 3, 4, 8])
def test_poisoned_self_exchange(oracle_mod, transport, period):
    P.test_self_exchange_ca_periods_bitwise(oracle_mod, transport, period)


@pytest.mark.parametrize("pg,n_local,L", [((2, 1, 1), (32, 32, 32), 3), ((2, 2, 2), (32, 32, 32), 3),
                                          ((1, 2, 3), (16, 32, 16), 2), ((2, 2, 1), (16, 16, 16), 2)])
@pytest.mark.parametrize("overlap", [True, False])
def test_poisoned_loopback(oracle_mod, pg, n_local, L, overlap):
    P.test_loopback_decomposition_bitwise(oracle_mod, pg, n_local, L, overlap)


@pytest.mark.parametrize("mode", ["loopback", "self-local", "self-nccl"])
def test_poisoned_pencil_overlap(oracle_mod, mode, monkeypatch):
    P.test_pencil_exchange_overlap_bitwise(oracle_mod, mode, monkeypatch)


@pytest.mark.parametrize("kw", [dict(ghost_mode=1, ca_period=3), dict(ghost_mode=1, ca_period=8),
                                dict(ghost_mode=1, ca_period=2, temporal_blocking=0)])
def test_poisoned_gsrb(oracle_mod, kw):
    P.test_gsrb_smoother_vcycle_bitwise(oracle_mod, kw)


@pytest.mark.parametrize("period", [1, 2, 3, 8])
@pytest.mark.parametrize("kernels", [(0, 3), (1, 0), (2, 0), (2, 1)])
def test_poisoned_bc_ca_periods_and_kernel_families(oracle_mod, period, kernels):
    V.test_bc_ca_periods_and_kernel_families_bitwise(oracle_mod, period, kernels)


@pytest.mark.parametrize("bc", [1, 2])
@pytest.mark.parametrize("pg,n_local,L", [((2, 1, 1), (32, 32, 32), 3), ((2, 2, 2), (32, 32, 32), 3)])
def test_poisoned_bc_loopback(oracle_mod, bc, pg, n_local, L):
    V.test_bc_loopback_decomposition_bitwise(oracle_mod, bc, pg, n_local, L, True)


@pytest.mark.parametrize("period", [1, 4, 8])
def test_poisoned_var_coef_ghost_shell(oracle_mod, period):
    V.test_var_coef_ca_periods_and_ghost_shells_bitwise(oracle_mod, period, 1)


@pytest.mark.parametrize("bc", [0, 1, 2])
def test_poisoned_var_coef_column_kernel(oracle_mod, bc):
    V.test_var_coef_column_kernel_bitwise(oracle_mod, bc, 1, 3)


@pytest.mark.parametrize("fusion", [1, 2, 3])
@pytest.mark.parametrize("period", [1, 3, 4])
@pytest.mark.parametrize("E", [4, 8])
def test_poisoned_fusion_ca_brick_edges(oracle_mod, fusion, period, E):
    V.test_brick4_fusion_ca_ghosts_bitwise(oracle_mod, fusion, period, 1, E)


@pytest.mark.parametrize("pg,n_local,L,bc", [((2, 1, 1), (16, 16, 16), 3, 0), ((2, 2, 2), (16, 16, 16), 2, 1)])
def test_poisoned_brick4_loopback(oracle_mod, pg, n_local, L, bc):
    V.test_brick4_loopback_decomposition_bitwise(oracle_mod, pg, n_local, L, bc)
